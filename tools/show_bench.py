"""Print the key fields of bench JSON lines: python tools/show_bench.py files..."""
import json, sys
for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "ERR", e); continue
    r = d.get("roofline", {})
    print(f"{f.split('/')[-1]:34s} algo={d.get('algo')} value={d['value']:.3e} ms={d['ms_per_step']:.4f} "
          f"stages={ {k: round(v, 4) for k, v in d.get('stage_ms', {}).items()} } frac={r.get('frac', 0):.3f} "
          f"best={d.get('result', {}).get('best')} clk={d.get('clocks', {}).get('sm_mhz')} e2e_ms={d.get('e2e', {}).get('ms_per_search', 0):.3f}")

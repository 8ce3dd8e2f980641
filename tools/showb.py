"""Print the key numbers of bench JSON lines: python tools/showb.py files..."""
import json, sys
for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        st = {k: round(v, 4) for k, v in d.get("stage_ms", {}).items()}
        e2e = d.get("e2e", {}).get("ms_per_search")
        print(f.split("/")[-1], round(d["ms_per_step"], 4), st, "e2e", e2e and round(e2e, 4),
              "best", d["result"]["best"], "frac", round(d["roofline"]["frac"], 4) if "roofline" in d else None)
    except Exception as e:
        print(f, "ERR", e)

"""Per-kernel durations from an ncu --metrics gpu__time_duration.sum CSV: python tools/launches.py file.csv"""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hdr]; ki = h.index("Kernel Name"); vi = h.index("Metric Value"); ui = h.index("Metric Unit")
agg = collections.OrderedDict()
for r in rows[hdr + 1:]:
    name = r[ki].split("(")[0][:60]
    v = float(r[vi].replace(",", ""))
    if r[ui] in ("nsecond", "ns"): v /= 1000.0
    elif r[ui] == "msecond": v *= 1000.0
    agg.setdefault(name, []).append(v)
tot = sum(sum(v) for v in agg.values())
for k, v in agg.items():
    print(f"{k:62s} n={len(v):3d} mean={sum(v)/len(v):10.2f} us  share={sum(v)/tot:6.3f}")

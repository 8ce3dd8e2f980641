"""Per-source-line instruction and stall-sample totals of one kernel in an
.ncu-rep (ncu --page source --print-source cuda,sass), normalised per unit.

    python tools/ncu_lines.py REP [--units U] [--top N]
"""
import argparse
import csv
import subprocess


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--units", type=float, default=1.0, help="divide instruction counts by this (e.g. warp-(row,b))")
    ap.add_argument("--top", type=int, default=40)
    a = ap.parse_args()
    out = subprocess.run(["ncu", "-i", a.rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    fname, lines, cur = None, {}, None
    hdr = None
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            fname = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            iW = hdr.index("Warp Stall Sampling (All Samples)")
            iE = hdr.index("Instructions Executed")
            continue
        if hdr is None or r[0] == "Function Name":
            continue
        if r[0]:  # a source line row (aggregated)
            cur = (fname, int(r[0]), r[1].strip())
            e = int(r[iE]) if r[iE].isdigit() else 0
            w = int(r[iW]) if r[iW].isdigit() else 0
            if e or w:
                d = lines.setdefault(cur, [0, 0])
                d[0] += e
                d[1] += w
    tot_e = sum(v[0] for v in lines.values())
    tot_w = sum(v[1] for v in lines.values())
    print(f"total instructions {tot_e} ({tot_e / a.units:.1f} per unit), stall samples {tot_w}")
    for (f, ln, src), (e, w) in sorted(lines.items(), key=lambda kv: -kv[1][0])[:a.top]:
        print(f"{f}:{ln:<5} {e / a.units:8.1f} {100 * e / tot_e:5.1f}%  stall {100 * w / max(tot_w, 1):5.1f}%  {src[:80]}")


if __name__ == "__main__":
    main()

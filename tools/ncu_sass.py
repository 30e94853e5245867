"""SASS of one kernel from an ncu report with per-instruction execution counts (address
order), to find where the warp instructions go.

usage: python tools/ncu_sass.py REPORT KERNEL_REGEX [--min COUNT]
"""
import csv
import io
import subprocess
import sys


def main():
    rep, kre = sys.argv[1], sys.argv[2]
    mn = float(sys.argv[sys.argv.index("--min") + 1]) if "--min" in sys.argv else 0
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", f"regex:{kre}",
                          "--launch-count", "1", "--print-source", "sass"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "Address"][0]
    h = rows[hi]
    ie, ss = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
    seen, recs = set(), []
    for r in rows[hi + 1:]:
        if len(r) <= ie or r[0] in seen:
            continue
        seen.add(r[0])
        try:
            recs.append((r[0], float(r[ie]), float(r[ss]), r[1].strip()))
        except ValueError:
            pass
    tot = sum(x[1] for x in recs)
    print(f"total warp instructions {tot:.0f}")
    for a, n, s, src in recs:
        if n >= mn:
            print(f"{a[-5:]} {n:12.0f} {100 * n / tot:5.2f}% {s:6.0f}  {src[:90]}")


if __name__ == "__main__":
    main()

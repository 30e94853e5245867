"""Top stall lines of one kernel from an ncu report (source page, SASS or CUDA source).

usage: python tools/ncu_hot.py REPORT KERNEL_REGEX [--cuda] [--top 25]
"""
import csv
import io
import subprocess
import sys


def main():
    rep, kre = sys.argv[1], sys.argv[2]
    cuda = "--cuda" in sys.argv
    top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 25
    cmd = ["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", f"regex:{kre}", "--launch-count", "1",
           "--print-source", "cuda" if cuda else "sass"]
    out = subprocess.run(cmd, capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hi = [i for i, r in enumerate(rows) if r and r[0] in ("Address", "Line", "#")][0]
    hdr = rows[hi]
    si = hdr.index("Warp Stall Sampling (All Samples)")
    src = hdr.index("Source")
    recs = []
    tot = 0
    seen = set()
    for r in rows[hi + 1:]:
        if len(r) <= si or r[0] in seen:      # one launch: each address once
            continue
        seen.add(r[0])
        try:
            v = float(r[si])
        except ValueError:
            continue
        tot += v
        recs.append((v, r[0], r[src].strip()))
    recs.sort(reverse=True)
    print(f"total samples {tot:.0f}")
    for v, a, s in recs[:top]:
        print(f"{100 * v / tot:5.1f}%  {a:>18}  {s[:110]}")


if __name__ == "__main__":
    main()

"""Per-source-line warp instructions and stall samples of one kernel from an ncu report
(--import-source on captures), summed over line ranges to attribute a kernel's
instructions to its phases.

usage: python tools/ncu_lines.py REPORT KERNEL_REGEX [FILE_SUBSTR] [--ranges a-b:name,...] [--top N]
"""
import csv
import io
import subprocess
import sys


def lines(rep, kre):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--kernel-name", f"regex:{kre}",
                          "--launch-count", "1", "--print-source", "cuda,sass"], capture_output=True,
                         text=True).stdout
    cur, recs = None, []
    ie = ss = None
    for r in csv.reader(io.StringIO(out)):
        if not r:
            continue
        if r[0] == "File Path":
            cur = r[1]
            continue
        if r[0] == "Line No":
            ie, ss = r.index("Instructions Executed"), r.index("Warp Stall Sampling (All Samples)")
            continue
        if r[0] and ie is not None and r[0].isdigit():
            try:
                recs.append((cur, int(r[0]), float(r[ie]), float(r[ss]), r[1].strip()))
            except ValueError:
                pass
    return recs


def main():
    rep, kre = sys.argv[1], sys.argv[2]
    fsub = sys.argv[3] if len(sys.argv) > 3 and not sys.argv[3].startswith("--") else ""
    recs = lines(rep, kre)
    tot = sum(x[2] for x in recs)
    stot = sum(x[3] for x in recs) or 1
    print(f"total warp instructions {tot:.0f}, stall samples {stot:.0f}")
    if "--ranges" in sys.argv:
        spec = sys.argv[sys.argv.index("--ranges") + 1]
        for part in spec.split(","):
            rng, name = part.split(":")
            a, b = map(int, rng.split("-"))
            n = sum(x[2] for x in recs if fsub in x[0] and a <= x[1] <= b)
            s = sum(x[3] for x in recs if fsub in x[0] and a <= x[1] <= b)
            print(f"{name:12s} {a:5d}-{b:5d} inst {n:12.0f} {100 * n / tot:5.1f}%  stalls {100 * s / stot:5.1f}%")
    top = int(sys.argv[sys.argv.index("--top") + 1]) if "--top" in sys.argv else 25
    for f, ln, n, s, src in sorted(recs, key=lambda x: -x[2])[:top]:
        print(f"{f.split('/')[-1]:14s}:{ln:<5d} {n:12.0f} {100 * n / tot:5.1f}% st {100 * s / stot:5.1f}%  {src[:80]}")


if __name__ == "__main__":
    main()

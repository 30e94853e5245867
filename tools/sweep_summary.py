"""Summarise sweep records (results/sweep2000_*.jsonl) as markdown tables: label
distributions overall, per nnz range and per generator family, infeasible formats.

usage: python tools/sweep_summary.py results/sweep2000_f64.jsonl [more.jsonl ...]
"""
import collections
import json
import sys


def dist(c):
    return ", ".join(f"{k} {v}" for k, v in c.most_common())


def summarise(path):
    recs = [json.loads(line) for line in open(path) if line.strip()]
    out = [f"### `{path.split('/')[-1]}`", ""]
    tot = sum(r["nnz"] for r in recs)
    agree = max(max((f.get("agree") or 0.0) for f in r["formats"].values() if isinstance(f, dict)) for r in recs)
    out.append(f"Matrices: {len(recs)}; total nonzeros {tot / 1e9:.2f} G; max cross-format disagreement "
               f"{agree:.1e} (relative to max|y|).")
    out += ["", "| label set | distribution |", "|---|---|"]
    for ls in ("label6", "label5", "label3"):
        out.append(f"| {ls} | {dist(collections.Counter(r[ls] for r in recs if r.get(ls)))} |")
    edges = [0, 10_000, 100_000, 1_000_000, 10_000_000, 10 ** 9]
    out += ["", "| nnz range | matrices | label6 distribution |", "|---|---|---|"]
    for lo, hi in zip(edges[:-1], edges[1:]):
        sel = [r for r in recs if lo <= r["nnz"] < hi]
        out.append(f"| [{lo:,}, {hi:,}) | {len(sel)} | {dist(collections.Counter(r['label6'] for r in sel))} |")
    out += ["", "| family | label6 distribution |", "|---|---|"]
    fams = collections.defaultdict(collections.Counter)
    for r in recs:
        fams[r["params"]["family"]][r["label6"]] += 1
    for f, c in fams.items():
        out.append(f"| {f} | {dist(c)} |")
    na = collections.Counter(f for r in recs for f, v in r["formats"].items() if isinstance(v, dict) and v.get("status") == "N/A")
    margins = sorted(r.get("margin") or 0.0 for r in recs)
    near = sum(1 for m in margins if m < 0.02)
    out += ["", f"Infeasible (A4, size guard): {dict(na)}. Winning margin t_2nd / t_best - 1: median "
                f"{margins[len(margins) // 2]:.3f}; {near} of {len(recs)} matrices are decided by less than 2%.", ""]
    return "\n".join(out)


if __name__ == "__main__":
    print("\n".join(summarise(p) for p in sys.argv[1:]))

"""Label reproducibility ("labels reproducible across two runs except
near-ties"): compare label6 of the matrices present in two sweep files.
usage: python tools/label_stability.py RUN1.jsonl RUN2.jsonl [--margin 0.02] [--out FILE]"""
import argparse
import json


def load(path):
    out = {}
    with open(path) as f:
        for line in f:
            r = json.loads(line)
            out[r["i"]] = r
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("a")
    ap.add_argument("b")
    ap.add_argument("--margin", type=float, default=0.02)
    ap.add_argument("--out", default="")
    a = ap.parse_args()
    A, B = load(a.a), load(a.b)
    common = sorted(set(A) & set(B))
    same = [i for i in common if A[i]["label6"] == B[i]["label6"]]
    clear = [i for i in common if min(A[i].get("margin") or 0, B[i].get("margin") or 0) >= a.margin]
    clear_same = [i for i in clear if A[i]["label6"] == B[i]["label6"]]
    flips = [{"i": i, "run1": A[i]["label6"], "run2": B[i]["label6"], "margin1": A[i].get("margin"),
              "margin2": B[i].get("margin"), "nnz": A[i]["nnz"]} for i in common if A[i]["label6"] != B[i]["label6"]]
    rep = {"matrices": len(common), "label6_agree": len(same), "label6_agree_frac": len(same) / max(1, len(common)),
           "margin_threshold": a.margin, "clear_matrices": len(clear), "clear_agree": len(clear_same),
           "clear_agree_frac": len(clear_same) / max(1, len(clear)),
           "flips_clear": [f for f in flips if f["i"] in set(clear)], "flips": flips[:50]}
    print(json.dumps({k: v for k, v in rep.items() if k not in ("flips",)}, indent=1))
    if a.out:
        with open(a.out, "w") as f:
            json.dump(rep, f, indent=1)


if __name__ == "__main__":
    main()

"""Summarise ncu outputs into tracked profiles/ files.

  python tools/ncu_summary.py launches  <launches.csv> <out.md>
  python tools/ncu_summary.py full      <report.ncu-rep> <out.md> [--traffic CONFIG DTYPE]

`launches` aggregates a `--metrics gpu__time_duration.sum` launch list per kernel
(count, mean, total, share).  `full` prints, per captured launch, duration, DRAM
bytes / throughput, L1/L2 hit rates, occupancy, registers and the top stall reasons;
with --traffic it also records DRAM bytes per launch of each format's SpMV kernel in
profiles/ncu_traffic.json (read by bench.py's roofline.traffic).
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def short(name):
    n = name.split("(")[0].replace("void ", "").replace("(anonymous namespace)::", "")
    n = n.replace("spmv::<unnamed>::", "").replace("<unnamed>::", "").strip()
    i = n.find("k_")
    if n.startswith("unnamed>::") or (i > 0 and "::" in n[:i]):
        n = n[i:]
    return n


SPMV_KERNELS = ("k_coo", "k_ell", "k_csr_vector", "k_csr_rows", "k_merge", "k_merge_persist", "k_merge_rows",
                "k_csr5")
B0_ARG = {"k_coo": 2, "k_ell": 1, "k_csr_vector": 3, "k_csr_rows": 2, "k_merge": 2, "k_merge_persist": 2,
          "k_merge_rows": 2, "k_csr5": 3}


def targs(name):
    return [a.strip() for a in name.split("<", 1)[1].rsplit(">", 1)[0].split(",")] if "<" in name else []


def is_beta0(name):
    """True for the beta == 0 instantiation of an SpMV kernel (not launched by a bench step)."""
    base, a = name.split("<")[0], targs(name)
    i = B0_ARG.get(base)
    return i is not None and i < len(a) and a[i] in ("1", "true")


def launches(path, out):
    rows = list(csv.reader(open(path)))
    i = [k for k, r in enumerate(rows) if "Kernel Name" in r][0]
    hdr = rows[i]
    agg = collections.OrderedDict()
    for r in rows[i + 1:]:
        d = dict(zip(hdr, r))
        if d.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(d["Metric Value"].replace(",", ""))
        unit = d["Metric Unit"]
        us = v / 1000 if unit == "ns" else (v * 1000 if unit == "ms" else v)
        agg.setdefault(short(d["Kernel Name"]), []).append(us)
    spmv = {k: v for k, v in agg.items() if k.startswith("k_")}
    tot = sum(sum(v) for v in spmv.values())
    with open(out, "w") as f:
        f.write(f"# ncu launch list summary: {os.path.basename(path)}\n\n")
        f.write("ncu --metrics gpu__time_duration.sum --clock-control none (serialised, cold-cache: compare "
                "shares, not absolutes)\n\n")
        f.write("| kernel | launches | mean us | total us | share of libspmv time |\n|---|---|---|---|---|\n")
        for k, v in agg.items():
            s = sum(v)
            share = f"{100 * s / tot:.1f}%" if k in spmv and tot else "-"
            f.write(f"| `{k}` | {len(v)} | {s / len(v):.1f} | {s:.1f} | {share} |\n")
        # share of one timed step: the step's SpMV launches (beta != 0 variants, fix-ups)
        # (ELL's kernel runs twice per step when HYB is all-ELL, as on LAP4096: K_h = K)
        step = {k: sum(v) / len(v) * (2 if k.startswith("k_ell<") else 1)
                for k, v in agg.items() if k.split("<")[0] in SPMV_KERNELS and not is_beta0(k)}
        fix = agg.get("k_fixup<double>") or agg.get("k_fixup<float>")
        if fix:
            step["k_fixup (x launches per step)"] = sum(fix) / len(fix) * 3
        st = sum(step.values())
        f.write("\n## Share of one bench step (mean launch time x launches per step)\n\n")
        f.write("| kernel | us per step | share |\n|---|---|---|\n")
        for k, v in sorted(step.items(), key=lambda kv: -kv[1]):
            f.write(f"| `{k}` | {v:.1f} | {100 * v / st:.1f}% |\n")
    print(open(out).read())


KEYS = [
    ("gpu__time_duration.sum", "time"),
    ("dram__bytes_read.sum", "dram_rd"),
    ("dram__bytes_write.sum", "dram_wr"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram%"),
    ("lts__t_sector_hit_rate.pct", "L2hit%"),
    ("l1tex__t_sector_hit_rate.pct", "L1hit%"),
    ("l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "L1thr%"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps%"),
    ("launch__registers_per_thread", "regs"),
    ("smsp__inst_executed.sum", "warp_inst"),
]


def to_bytes(v, unit):
    m = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
    return float(v.replace(",", "")) * m.get(unit, 1)


def full(rep, out, traffic=None, formats=("coo", "ell", "csr", "hyb", "merge", "csr5")):
    """Per launch: duration, DRAM bytes, hit rates, occupancy, registers, top stalls.  With a
    capture taken under --nvtx (tools/prof_formats.py: one spmv_run per format inside
    libspmv's own "spmv_run:<fmt>" ranges), every kernel of a run -- the chunk and row
    kernels of CSR, merge's two tile kernels, the fix-ups -- is attributed to its format
    by the range, and the traffic per run is their sum."""
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(raw)))
    hdr, units = r[0], r[1]
    nv = [h for h in hdr if h.startswith("thread Domain:Push/Pop_Range")]
    pre = "smsp__average_warps_issue_stalled_"
    lines = [f"# ncu --set full summary: {os.path.basename(rep)}\n",
             "ncu --set full --clock-control none --import-source on --nvtx (one replayed launch per row; "
             "DRAM bytes attributed to the spmv_run:<format> NVTX range each kernel ran in)\n",
             "| range | kernel | " + " | ".join(k[1] for k in KEYS) + " | top stalls (warps per issue) |",
             "|---|---|" + "---|" * (len(KEYS) + 1)]
    trafficmap = collections.OrderedDict()
    for row in r[2:]:
        d = dict(zip(hdr, row))
        name = short(d["Kernel Name"])
        rng = ""
        if nv:
            m = d.get(nv[0], "")
            i = m.find("<default domain>:")
            rng = m[i + len("<default domain>:"):].split(":none")[0] if i >= 0 else ""
        cells = []
        for k, _ in KEYS:
            u = units[hdr.index(k)] if k in hdr else ""
            cells.append(f"{d.get(k, '')} {u}".strip())
        st = {h[len(pre):].replace("_per_issue_active.ratio", ""): float(d[h]) for h in hdr
              if h.startswith(pre) and h.endswith("_per_issue_active.ratio") and d[h] not in ("", "n/a")}
        top = ", ".join(f"{k} {v:.1f}" for v, k in sorted(((v, k) for k, v in st.items()), reverse=True)[:3])
        lines.append(f"| {rng} | `{name}` | " + " | ".join(cells) + f" | {top} |")
        key = rng.replace("spmv_run:", "") if rng.startswith("spmv_run:") else ("features" if "features" in rng
                                                                                 else None)
        if key:
            rd = to_bytes(d["dram__bytes_read.sum"], units[hdr.index("dram__bytes_read.sum")])
            wr = to_bytes(d["dram__bytes_write.sum"], units[hdr.index("dram__bytes_write.sum")])
            trafficmap[key] = trafficmap.get(key, 0) + rd + wr
    if trafficmap:
        lines += ["", "## DRAM bytes per run (all kernels of the range)", "",
                  "| range | DRAM bytes (read+write) |", "|---|---|"]
        lines += [f"| {k} | {v:.4g} |" for k, v in trafficmap.items()]
    with open(out, "w") as f:
        f.write("\n".join(lines) + "\n")
    print("\n".join(lines))
    if traffic:
        cfg, dt = traffic
        p = os.environ.get("NCU_TRAFFIC_JSON", os.path.join(ROOT, "profiles", "ncu_traffic.json"))
        d = json.load(open(p)) if os.path.exists(p) else {}
        d.setdefault(cfg, {})[dt] = {k: int(v) for k, v in trafficmap.items()}
        d["_note"] = ("DRAM bytes (read+write) of one spmv_run of each format -- every kernel of the run, "
                      "attributed by libspmv's spmv_run:<format> NVTX range -- and of one spmv_features call, from "
                      "one ncu --set full --nvtx capture of tools/prof_formats.py; see profiles/*.md")
        json.dump(d, open(p, "w"), indent=1, sort_keys=True)
        print("traffic:", dict(trafficmap))


if __name__ == "__main__":
    mode = sys.argv[1]
    if mode == "launches":
        launches(sys.argv[2], sys.argv[3])
    else:
        tr = None
        if "--traffic" in sys.argv:
            i = sys.argv.index("--traffic")
            tr = (sys.argv[i + 1], sys.argv[i + 2])
        fm = ("coo", "ell", "csr", "hyb", "merge", "csr5")
        if "--formats" in sys.argv:
            fm = tuple(sys.argv[sys.argv.index("--formats") + 1].split(","))
        full(sys.argv[2], sys.argv[3], tr, fm)

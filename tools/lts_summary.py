"""Summarise ncu --metrics CSV launch lists (L2/LTS, L1, DRAM throughput per kernel) into a
markdown table; kernels attributed to formats by NVTX range when present.
usage: python tools/lts_summary.py CSV [CSV ...] > out.md"""
import csv
import sys


def rows(path):
    lines = open(path).read().splitlines()
    i = [k for k, l in enumerate(lines) if l.startswith('"ID"')][0]
    r = list(csv.reader(lines[i:]))
    hdr = r[0]
    out = {}
    nv = [h for h in hdr if h.startswith("thread Domain:Push/Pop_Range")]
    for row in r[1:]:
        d = dict(zip(hdr, row))
        key = (d["ID"], d["Kernel Name"].split("(")[0].replace("void ", "").split("::")[-1][:40])
        rng = ""
        if nv and d.get(nv[0]):
            m = d[nv[0]]
            j = m.find("<default domain>:")
            rng = m[j + 17:].split(":none")[0] if j >= 0 else ""
        e = out.setdefault(key, {"range": rng})
        e[d["Metric Name"]] = (d["Metric Value"].replace(",", ""), d["Metric Unit"])
    return out


COLS = [("gpu__time_duration.sum", "time"), ("lts__t_sectors.avg.pct_of_peak_sustained_elapsed", "LTS sectors %peak"),
        ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "LTS thr %"), ("lts__t_sectors.sum", "LTS sectors"),
        ("lts__t_sector_hit_rate.pct", "L2 hit %"), ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM %"),
        ("dram__bytes_read.sum", "DRAM rd"), ("l1tex__throughput.avg.pct_of_peak_sustained_elapsed", "L1 thr %"),
        ("l1tex__t_sector_hit_rate.pct", "L1 hit %"), ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "ld requests"),
        ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "ld sectors"),
        ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps %")]


def main():
    for p in sys.argv[1:]:
        print(f"\n### {p.split('/')[-1]}\n")
        print("| range | kernel | " + " | ".join(c[1] for c in COLS) + " |")
        print("|---|---|" + "---|" * len(COLS))
        for (i, k), e in rows(p).items():
            cells = []
            for m, _ in COLS:
                v = e.get(m)
                cells.append(f"{v[0]} {v[1]}".strip() if v else "")
            print(f"| {e['range']} | `{k}` | " + " | ".join(cells) + " |")


if __name__ == "__main__":
    main()

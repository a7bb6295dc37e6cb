#!/usr/bin/env python
"""Summarise ncu output (from tools/profile.sh) into a markdown file for profiles/.

    python tools/ncu_summary.py gpurun_out profiles/r01_ncu_summary.md

Reads gpurun_out/launches.csv (gpu__time_duration.sum per launch) and every
gpurun_out/prof_*.ncu-rep (--set full) via `ncu -i ... --page raw --csv`.
"""
import csv
import glob
import io
import os
import subprocess
import sys
from collections import defaultdict

RAW_KEYS = [
    ("gpu__time_duration.sum", "time"),
    ("dram__bytes_read.sum", "dram rd"),
    ("dram__bytes_write.sum", "dram wr"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram %peak"),
    ("lts__t_sector_hit_rate.pct", "L2 hit %"),
    ("l1tex__t_sector_hit_rate.pct", "L1 hit %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM %peak"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
]


def short(name: str) -> str:
    name = name.replace("void ", "")
    base = name.split("(")[0]
    return base.replace("xbfs::", "").replace("<unnamed>::", "")[:60]


def launches(path):
    rows = list(csv.reader(open(path)))
    h = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    hdr = rows[h]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = defaultdict(lambda: [0, 0.0])
    for r in rows[h + 1:]:
        if len(r) <= vi:
            continue
        try:
            v = float(r[vi].replace(",", ""))
        except ValueError:
            continue
        scale = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "nsecond": 1e-3, "ms": 1e3, "msecond": 1e3}.get(r[ui], 1e-3)
        a = agg[short(r[ki])]
        a[0] += 1
        a[1] += v * scale
    return agg


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return [], []
    hdr, units = rows[0], rows[1]
    recs = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        recs.append({"kernel": short(d.get("Kernel Name", "?")),
                     **{lab: (d.get(k, ""), u.get(k, "")) for k, lab in RAW_KEYS}})
    return recs, [lab for _, lab in RAW_KEYS]


def main():
    src, dst = sys.argv[1], sys.argv[2]
    title = sys.argv[3] if len(sys.argv) > 3 else "ncu summary"
    lines = [f"# {title}", ""]
    lp = os.path.join(src, "launches.csv")
    if os.path.exists(lp):
        agg = launches(lp)
        def is_bfs(k):   # the library's BFS kernels (not the CSR build, stats, CUB / torch validation kernels)
            return k.startswith("k_") and all(s not in k for s in (
                "reorder", "check_and_pack", "split_keys", "degree_facts", "count_m", "k_head"))
        tot_bfs = sum(t for k, (n, t) in agg.items() if is_bfs(k))
        lines += ["## Launch list (`ncu --metrics gpu__time_duration.sum --clock-control none`)", "",
                  "Cold-cache, serialised per-launch times: compare SHARES, not absolutes.  `share` is of the BFS",
                  "kernels only (CSR build / reorder / stats / torch fill kernels excluded).", "",
                  "| kernel | launches | total us | avg us | share of BFS |", "|---|---|---|---|---|"]
        for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
            bfs = is_bfs(k)
            share = f"{100 * t / tot_bfs:.1f}%" if bfs and tot_bfs else "-"
            lines.append(f"| `{k}` | {n} | {t:.1f} | {t / n:.2f} | {share} |")
        lines.append("")
    for rep in sorted(glob.glob(os.path.join(src, "prof_*.ncu-rep"))):
        recs, labs = raw(rep)
        if not recs:
            continue
        lines += [f"## `{os.path.basename(rep)}` (`--set full`)", "",
                  "| kernel | " + " | ".join(labs) + " |", "|---" * (len(labs) + 1) + "|"]
        for r in recs:
            cells = []
            for lab in labs:
                v, u = r[lab]
                cells.append(f"{v} {u}".strip())
            lines.append(f"| `{r['kernel']}` | " + " | ".join(cells) + " |")
        lines.append("")
    open(dst, "w").write("\n".join(lines) + "\n")
    print(dst)


if __name__ == "__main__":
    main()

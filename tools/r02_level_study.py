#!/usr/bin/env python
"""Per-level, per-strategy study on B200 (the paper's Tabs III-VI,
P:L233-343, measured on R25 = Kronecker scale 25): for every level k of a BFS,
run level k with each strategy SF / SS / BU (levels before k follow the
adaptive choice, levels after k go back to the selector) through the host-loop
driver, which launches one kernel per phase so that ncu can attribute DRAM
bytes, L2 hit rate and time to (level, strategy).

    python tools/r02_level_study.py --config s25 --roots 1 --out gpurun_out/ls_s25.json
    ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,\
lts__t_sector_hit_rate.pct --csv --log-file gpurun_out/ls_ncu.csv python tools/r02_level_study.py ...
    python tools/r02_level_study.py --report gpurun_out/ls_s25.json --ncu gpurun_out/ls_ncu.csv > profiles/...md

The JSON records every run's launch sequence (kernel, level) so the ncu rows can
be matched launch by launch; D-3 algorithmic bytes per level come
from the run's own per-level counters.
"""
import argparse
import csv
import io
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

NAMES = {0: "SF", 1: "SS", 2: "BU"}
OUR_KERNELS = ("k_init_fill", "k_seed", "k_generate", "k_td_expand", "k_ss_count", "k_bu_traverse", "k_select",
               "k_small_sf")


def measure(args):
    import numpy as np
    import torch

    import bench
    from paper_conf_sc_yangls0w24_b200 import metrics
    from paper_conf_sc_yangls0w24_b200.xbfs import Graph
    torch.cuda.set_device(0)
    src, dst, n = bench.make_graph(args.config, pinned=True)
    roots = bench.pick_roots(args.config, n, src, dst, args.roots + 1)
    g = Graph(torch.from_numpy(src.view(np.int32)), torch.from_numpy(dst.view(np.int32)), n)
    level = torch.empty(n, dtype=torch.int32, device="cuda")
    parent = torch.empty(n, dtype=torch.int32, device="cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    runs = []

    def run(root, tag, **kw):
        flush.fill_(1)
        torch.cuda.synchronize()
        _, _, st = g.run(int(root), level, parent, stats=True, profile=4096, driver=1, small_edges=0, **kw)
        d3 = metrics.d3_level_bytes(n, st.strategy, st.frontier_vertices, st.frontier_edges, st.unvisited,
                                    st.bu_probes)
        runs.append({"tag": tag, "root": int(root), "strategy": st.strategy, "fv": st.frontier_vertices,
                     "fe": st.frontier_edges, "unvisited": st.unvisited, "probes": st.bu_probes, "d3": d3,
                     "launches": [(name, lvl, ms) for (name, lvl, ms) in st.kernels]})
        return st

    run(roots[0], "warmup")
    for root in roots[1:]:
        base = run(root, "adaptive")
        adaptive = list(base.strategy)
        for k in range(base.num_levels):
            for s in (0, 1, 2):
                run(root, f"L{k}:{NAMES[s]}", plan=adaptive[:k] + [s])
    json.dump({"config": bench.workload_name(args.config), "n": n, "arcs": g.arcs, "runs": runs},
              open(args.out, "w"))


def report(args):
    d = json.load(open(args.report))
    if args.timing:   # event times from a run outside ncu (same launch sequence)
        tmg = json.load(open(args.timing))
        for r, t in zip(d["runs"], tmg["runs"]):
            assert [x[:2] for x in r["launches"]] == [x[:2] for x in t["launches"]], r["tag"]
            r["launches"] = t["launches"]
    rows = []
    if args.ncu:
        txt = open(args.ncu).read()
        body = txt[txt.index('"ID"'):]
        recs = list(csv.DictReader(io.StringIO(body)))
        per = {}
        order = []
        for r in recs:
            kid = r["ID"]
            if kid not in per:
                per[kid] = {"name": r["Kernel Name"]}
                order.append(kid)
            per[kid][r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
        rows = [per[i] for i in order if any(per[i]["name"].split("(")[0].split("<")[0].endswith(k)
                                            for k in OUR_KERNELS)]
        nl = sum(len(r["launches"]) for r in d["runs"])
        rows = rows[-nl:]
        assert len(rows) == nl, (len(rows), nl)
    it = iter(rows)
    arcs = d["arcs"]
    out = [f"# Per-level strategy study on B200 ({d['config']}, A = {arcs:,} arcs)", ""]
    out.append("Host-loop driver (one launch per phase, so ncu attributes counters per level); each level k "
               "forced to SF / SS / BU with the adaptive choice before it.  ms = sum of the level's "
               "CUDA-event-timed launches; D-3 MB = SURVEY §8(d) algorithmic bytes of level k; DRAM MB / L2 hit "
               "= ncu `dram__bytes_read.sum + dram__bytes_write.sum` and `lts__t_sector_hit_rate.pct` of the "
               "level's launches (cold-cache, serialised replay).  The paper's Tabs III-VI (P:L233-343) are "
               "the same table on MI250X / R25.")
    out.append("")
    by_root = {}
    for r in d["runs"]:
        launches = r["launches"]
        ncu = [next(it) for _ in launches] if rows else [None] * len(launches)
        lv = {}
        for (name, k, ms), m in zip(launches, ncu):
            if k < 0:
                continue
            e = lv.setdefault(k, {"ms": 0.0, "dram": 0.0, "hit_w": 0.0, "t": 0.0})
            e["ms"] += ms
            if m:
                e["dram"] += m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
                dt = m.get("gpu__time_duration.sum", 0)
                e["hit_w"] += m.get("lts__t_sector_hit_rate.pct", 0) * dt
                e["t"] += dt
        r["lv"] = lv
        if r["tag"] != "warmup":
            by_root.setdefault(r["root"], []).append(r)
    for root, rs in by_root.items():
        base = rs[0]
        out.append(f"## root {root} (adaptive: {''.join('FSB'[s] for s in base['strategy'])})")
        out.append("")
        out.append("| level | ratio | \\|F\\| | strategy | ms | D-3 MB | DRAM MB | L2 hit % | BU probes | adaptive |")
        out.append("|---|---|---|---|---|---|---|---|---|---|")
        for r in rs[1:]:
            k = int(r["tag"][1:].split(":")[0])
            sname = r["tag"].split(":")[1]
            e = r["lv"].get(k, {"ms": 0, "dram": 0, "hit_w": 0, "t": 0})
            hit = e["hit_w"] / e["t"] if e["t"] else float("nan")
            out.append(f"| {k} | {base['fe'][k] / arcs:.3g} | {base['fv'][k]:,} | {sname} | {e['ms']:.4f} | "
                       f"{r['d3'][k] / 1e6:.2f} | {e['dram'] / 1e6:.2f} | {hit:.1f} | "
                       f"{r['probes'][k]:,} | {'yes' if NAMES[base['strategy'][k]] == sname else ''} |")
        out.append("")
    print("\n".join(out))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="s25")
    ap.add_argument("--roots", type=int, default=1)
    ap.add_argument("--out", default="gpurun_out/ls.json")
    ap.add_argument("--report", default=None)
    ap.add_argument("--ncu", default=None)
    ap.add_argument("--timing", default=None, help="JSON of a run outside ncu: its event times are reported")
    args = ap.parse_args()
    if args.report:
        report(args)
    else:
        measure(args)


if __name__ == "__main__":
    main()

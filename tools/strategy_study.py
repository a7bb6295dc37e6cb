#!/usr/bin/env python
"""B200 replay of the paper's strategy study.

* Tab VI analogue: for every level k of a BFS, run level k with
  each strategy SF / SS / BU (levels before k follow the adaptive choice, levels
  after k go back to the selector) and report level k's device time (sum of its
  event-timed launches) and algorithmic bytes.  Fig 7 / alpha: the
  ratio at which BU starts to win.
* Tab I analogue: per-level time and BU probes with the
  degree-aware neighbour re-arrangement on and off.

    python tools/strategy_study.py --config s24 --roots 2 --out profiles/r01_strategy_study
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_sc_yangls0w24_b200.xbfs import Graph  # noqa: E402

NAMES = {0: "SF", 1: "SS", 2: "BU"}


def level_times(st, n):
    per = {}
    byt = {}
    for name, lvl, ms in st.kernels:
        if lvl < 0:
            continue
        per[lvl] = per.get(lvl, 0.0) + ms
        byt[lvl] = byt.get(lvl, 0) + bench.kernel_bytes(name, lvl, st, n)
    return per, byt


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="s24")
    ap.add_argument("--roots", type=int, default=2)
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    torch.cuda.set_device(0)
    src, dst, n = bench.make_graph(args.config, pinned=True)
    roots = bench.pick_roots(args.config, n, src, dst, args.roots + 2)
    g = Graph(torch.from_numpy(src.view(np.int32)), torch.from_numpy(dst.view(np.int32)), n)
    level = torch.empty(n, dtype=torch.int32, device="cuda")
    parent = torch.empty(n, dtype=torch.int32, device="cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")

    def run(root, **kw):
        flush.fill_(1)
        torch.cuda.synchronize()
        _, _, st = g.run(int(root), level, parent, stats=True, profile=8192, driver=1, **kw)
        return st

    for r in roots[:2]:
        run(r)                                                    # warm-up
    study = {"config": bench.workload_name(args.config), "n": n, "arcs": g.arcs, "roots": []}
    for root in roots[2:]:
        base = run(root)
        adaptive = list(base.strategy)
        t_base, b_base = level_times(base, n)
        rows = []
        for k in range(base.num_levels):
            row = {"level": k, "ratio": base.frontier_edges[k] / g.arcs, "frontier": base.frontier_vertices[k],
                   "adaptive": NAMES[adaptive[k]]}
            for s in (0, 1, 2):
                st = run(root, plan=adaptive[:k] + [s], small_edges=0)
                assert st.num_levels == base.num_levels
                t, b = level_times(st, n)
                row[NAMES[s] + "_ms"] = round(t.get(k, 0.0), 4)
                row[NAMES[s] + "_MB"] = round(b.get(k, 0) / 1e6, 2)
                if s == 2:
                    row["BU_probes"] = st.bu_probes[k]
            row["best"] = min(("SF", "SS", "BU"), key=lambda x: row[x + "_ms"])
            rows.append(row)
        # Tab I analogue: re-arrangement off vs on (adaptive strategies of the re-arranged run)
        g.reorder(0)
        off = run(root, plan=adaptive, small_edges=0)
        g.reorder(1)
        on = run(root, plan=adaptive, small_edges=0)
        t_off, _ = level_times(off, n)
        t_on, _ = level_times(on, n)
        tab1 = [{"level": k, "strategy": NAMES[adaptive[k]], "ms_not_rearranged": round(t_off.get(k, 0), 4),
                 "ms_rearranged": round(t_on.get(k, 0), 4), "bu_probes_not_rearranged": off.bu_probes[k],
                 "bu_probes_rearranged": on.bu_probes[k]} for k in range(base.num_levels)]
        study["roots"].append({"root": int(root), "levels": rows, "tab1": tab1,
                               "total_ms_not_rearranged": round(off.elapsed_ms, 4),
                               "total_ms_rearranged": round(on.elapsed_ms, 4)})
        print(json.dumps(study["roots"][-1]), flush=True)
    if args.out:
        json.dump(study, open(args.out + ".json", "w"), indent=1)
        lines = [f"# Strategy study on B200 ({study['config']}, A = {study['arcs']:,} arcs)", "",
                 "Per-level device time (ms, sum of the level's CUDA-event-timed launches, host-loop driver) and",
                 "algorithmic MB with each strategy forced at that level only; the paper's Table VI (P:L320-343)",
                 "measured the same on MI250X / R25.  `adaptive` = this build's selector (alpha 0.1, BU",
                 "hysteresis 1.0).", ""]
        for r in study["roots"]:
            lines += [f"## root {r['root']}", "",
                      "| level | ratio | |F| | SF ms | SS ms | BU ms | best | adaptive | SF MB | SS MB | BU MB | BU probes |",
                      "|---|---|---|---|---|---|---|---|---|---|---|---|"]
            for x in r["levels"]:
                lines.append(f"| {x['level']} | {x['ratio']:.3g} | {x['frontier']:,} | {x['SF_ms']} | {x['SS_ms']} | "
                             f"{x['BU_ms']} | {x['best']} | {x['adaptive']} | {x['SF_MB']} | {x['SS_MB']} | "
                             f"{x['BU_MB']} | {x['BU_probes']:,} |")
            lines += ["", f"Re-arrangement (Tab I analogue, P:L155-171): total {r['total_ms_not_rearranged']} ms "
                      f"not re-arranged vs {r['total_ms_rearranged']} ms re-arranged", "",
                      "| level | strategy | ms not re-arranged | ms re-arranged | BU probes not | BU probes re-arranged |",
                      "|---|---|---|---|---|---|"]
            for x in r["tab1"]:
                lines.append(f"| {x['level']} | {x['strategy']} | {x['ms_not_rearranged']} | {x['ms_rearranged']} | "
                             f"{x['bu_probes_not_rearranged']:,} | {x['bu_probes_rearranged']:,} |")
            lines.append("")
        open(args.out + ".md", "w").write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()

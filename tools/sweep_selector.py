#!/usr/bin/env python
"""Selector sweep on B200 (the paper's alpha study P:L214-225 /
Tab VI P:L320-343 replayed): GTEPS of the adaptive BFS for a grid of
(alpha, bu_stay, grow) values on one Kronecker graph, same roots for all.

    python tools/sweep_selector.py --config s24 --roots 16
"""
import argparse
import itertools
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_sc_yangls0w24_b200 import metrics  # noqa: E402
from paper_conf_sc_yangls0w24_b200.xbfs import Graph  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="s24")
    ap.add_argument("--roots", type=int, default=16)
    ap.add_argument("--alphas", default="0.2,0.1,0.05,0.03,0.02,0.01")
    ap.add_argument("--stays", default="0,0.25,1,4")
    ap.add_argument("--grows", default="2.0")
    ap.add_argument("--driver", type=int, default=0)
    args = ap.parse_args()
    torch.cuda.set_device(0)
    src, dst, n = bench.make_graph(args.config, pinned=True)
    roots = bench.pick_roots(args.config, n, src, dst, args.roots + 3)
    g = Graph(torch.from_numpy(src.view(np.int32)), torch.from_numpy(dst.view(np.int32)), n)
    level = torch.empty(n, dtype=torch.int32, device="cuda")
    parent = torch.empty(n, dtype=torch.int32, device="cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for r in roots[:3]:
        g.run(int(r), level, parent, stats=True)
    out = []
    for a, b, gr in itertools.product([float(x) for x in args.alphas.split(",")],
                                      [float(x) for x in args.stays.split(",")],
                                      [float(x) for x in args.grows.split(",")]):
        teps, ms, strat = [], [], []
        for r in roots[3:]:
            flush.fill_(1)
            _, _, st = g.run(int(r), level, parent, stats=True, alpha=a, bu_stay=b, grow=gr, driver=args.driver)
            teps.append(st.input_edges_traversed / (st.elapsed_ms * 1e-3))
            ms.append(st.elapsed_ms)
            strat.append("".join("FSB"[s] for s in st.strategy))
        rec = {"alpha": a, "bu_stay": b, "grow": gr, "gteps_hmean": round(metrics.harmonic_mean(teps) / 1e9, 2),
               "ms_mean": round(float(np.mean(ms)), 4), "strategies": sorted(set(strat))[:4]}
        out.append(rec)
        print(json.dumps(rec), flush=True)
    best = max(out, key=lambda r: r["gteps_hmean"])
    print("BEST", json.dumps(best))


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""Per-level device time of the persistent driver (%globaltimer stamps) for a few
s24 roots: strategy, |F_k|, edgesF_k / A, |U_k|, BU probes, us.

    python tools/level_times.py [--config s24] [--roots 4] [extra run opts as k=v ...]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_sc_yangls0w24_b200.xbfs import Graph  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="s24")
    ap.add_argument("--roots", type=int, default=4)
    ap.add_argument("opts", nargs="*")
    args = ap.parse_args()
    opts = {}
    for kv in args.opts:
        k, v = kv.split("=")
        opts[k] = float(v) if "." in v else int(v)
    torch.cuda.set_device(0)
    src, dst, n = bench.make_graph(args.config, pinned=True)
    roots = bench.pick_roots(args.config, n, src, dst, args.roots + 3)
    g = Graph(torch.from_numpy(src.view(np.int32)), torch.from_numpy(dst.view(np.int32)), n)
    level = torch.empty(n, dtype=torch.int32, device="cuda")
    parent = torch.empty(n, dtype=torch.int32, device="cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for r in roots[:3]:
        g.run(int(r), level, parent, stats=True, **opts)
    for r in roots[3:]:
        flush.fill_(1)
        torch.cuda.synchronize()
        _, _, st = g.run(int(r), level, parent, stats=True, **opts)
        print(f"root {int(r)}: {st.elapsed_ms * 1e3:.1f} us total, levels sum {sum(st.level_ms) * 1e3:.1f} us, "
              f"init {st.init_ms * 1e3:.1f} us")
        for k in range(st.num_levels):
            print(f"  L{k} {'FSB'[st.strategy[k]]} |F|={st.frontier_vertices[k]:>9,} ratio={st.frontier_edges[k] / g.arcs:9.3g} "
                  f"U={st.unvisited[k]:>10,} probes={st.bu_probes[k]:>11,} {st.level_ms[k] * 1e3:8.1f} us")


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""Per-level fixed cost on B200: device time per BFS level of tiny graphs (where
the level kernels do ~no work) for each driver and forced strategy, plus the s24
per-root elapsed time under both drivers.  Latency evidence for DESIGN.md §5.

    python tools/level_floor.py
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
from paper_conf_sc_yangls0w24_b200.xbfs import Graph  # noqa: E402


def path_graph(n):
    src = np.arange(n - 1, dtype=np.int32)
    return src, src + 1, n


def per_level(g, root, reps=5, **kw):
    out = []
    for _ in range(reps):
        _, _, st = g.run(root, stats=True, **kw)
        out.append(st.elapsed_ms / max(st.num_levels, 1))
    return float(np.median(out)) * 1e3, st.num_levels


def main():
    torch.cuda.set_device(0)
    res = {}
    for n in (64, 4096):
        src, dst, nn = path_graph(n)
        g = Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), nn)
        for drv in (1, 2, 3):
            for force, small in ((-1, 0), (0, 0), (1, 0), (2, 0), (-1, 65536)):
                if (n > 64 and force == 2) or (drv == 3 and small):
                    continue
                us, nl = per_level(g, 0, driver=drv, force_strategy=force, small_edges=small)
                key = f"path{n} driver{drv} force{force} small{small}"
                res[key] = {"us_per_level": round(us, 2), "levels": nl}
                print(key, res[key], flush=True)
        g.close()
    src, dst, n = bench.make_graph("s24", pinned=True)
    roots = bench.pick_roots("s24", n, src, dst, 12)
    g = Graph(torch.from_numpy(src.view(np.int32)), torch.from_numpy(dst.view(np.int32)), n)
    level = torch.empty(n, dtype=torch.int32, device="cuda")
    parent = torch.empty(n, dtype=torch.int32, device="cuda")
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for drv in (1, 2, 3):
        for r in roots[:3]:
            g.run(int(r), level, parent, stats=True, driver=drv)
        rows = []
        for r in roots[3:]:
            flush.fill_(1)
            _, _, st = g.run(int(r), level, parent, stats=True, driver=drv)
            rows.append((int(r), round(st.elapsed_ms, 4), "".join("FSB"[s] for s in st.strategy)))
        res[f"s24 driver{drv}"] = rows
        print(f"s24 driver{drv}", rows, "mean", np.mean([x[1] for x in rows]), flush=True)
    json.dump(res, open(os.path.join(ROOT, "gpurun_out", "level_floor.json"), "w"), indent=1)


if __name__ == "__main__":
    main()

"""Directed-graph scale sweep on the GPU (debug): build, run every root under the
adaptive selector, forced BU and forced SF, and check the three level arrays agree
(parity against the oracle lives in tests/test_directed_gpu.py)."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from paper_conf_sc_yangls0w24_b200 import synth
from paper_conf_sc_yangls0w24_b200.xbfs import Graph

undirected = os.environ.get("UNDIRECTED") == "1"
for scale in [int(x) for x in sys.argv[1:]] or [16, 18, 20, 22, 24]:
    src, dst, n = synth.kronecker(scale, seed=1)
    t0 = time.time()
    g = Graph(src, dst, n, directed=not undirected)
    torch.cuda.synchronize()
    print(f"s{scale}: built {time.time()-t0:.1f}s arcs {g.arcs} maxdeg {g.max_degree}", flush=True)
    for r in synth.roots(n, src, dst, 6):
        first = None
        for opts in (dict(), dict(force_strategy=2), dict(force_strategy=0), dict(force_strategy=1),
                     dict(force_strategy=0, driver=1)):
            if opts.get("driver") == 1 and not undirected:
                continue
            lv, pa, st = g.run(int(r), stats=True, **opts)
            torch.cuda.synchronize()
            msg = f"  root {r} {opts} levels {st.num_levels} reached {st.vertices_reached} ms {st.elapsed_ms:.3f} " \
                  f"strat {''.join('FSB'[s] for s in st.strategy)}"
            if first is None:
                first = lv.clone()
            msg += f" same {bool(torch.equal(first, lv))}"
            print(msg, flush=True)
    g.close()

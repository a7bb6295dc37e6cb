"""Multi-GPU path (include/xbfs_dist.h) on the GPU: `world` processes share
cuda:0 (CUDA IPC maps each rank's replicas, inbox and build buffers into the
peers exactly as across NVLink peers); the communicator is the library's own
(unique id broadcast over gloo).  Every rank passes only ITS share of the input
tuples to xbfs_build_csr_dist.  Gathered levels must equal the oracle
bit-exactly; parents must pass Graph500 validation and, where a bottom-up step
found the vertex, equal reading R-12's parent (the first vertex of the
re-arranged row one level up: the partition's rows are xbfs_reorder's rows) —
for the adaptive selector and every strategy forced on every level.  The
per-level counters and Graph500 m are global and must equal the oracle's."""
import os
import socket

import numpy as np
import pytest

import oracle
from paper_conf_sc_yangls0w24_b200 import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

MODES = [dict(), dict(force_strategy=0), dict(force_strategy=1), dict(force_strategy=2), dict(alpha=0.02),
         dict(bu_stay=0.0)]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, graph, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        from paper_conf_sc_yangls0w24_b200.dist import Comm, DistGraph, tuple_range
        src, dst, n = _graph(graph)
        e0, e1 = tuple_range(src.shape[0], world, rank)
        comm = Comm.from_torch()
        on_dev = rank % 2 == 1                      # host and device tuple shares mixed
        s_, d_ = src[e0:e1].copy(), dst[e0:e1].copy()
        if on_dev:
            s_ = torch.from_numpy(s_.view(np.int32)).cuda()
            d_ = torch.from_numpy(d_.view(np.int32)).cuda()
        dg = DistGraph(comm, s_, d_, n)
        assert dg.n == n and dg.m_input == src.shape[0]
        roots = synth.roots(n, src, dst, 4, root_seed=11).tolist() + [0]
        out = []
        for root in roots:
            for mi, opts in enumerate(MODES):
                lv, pa, st = dg.run(int(root), **opts)
                lvs, pas = [None] * world, [None] * world
                dist.all_gather_object(lvs, lv.cpu().numpy())
                dist.all_gather_object(pas, pa.cpu().numpy())
                if rank == 0:
                    out.append((int(root), mi, np.concatenate(lvs), np.concatenate(pas), st.strategy,
                                st.frontier_vertices, st.frontier_edges, st.unvisited, st.input_edges_traversed,
                                st.num_levels, dg.arcs))
        dg.close()
        comm.close()
        q.put((rank, out))
    except Exception as e:
        import traceback
        q.put((rank, f"{type(e).__name__}: {e}\n{traceback.format_exc()}"))
    finally:
        dist.destroy_process_group()


def _graph(name):
    if name == "kron":
        return synth.kronecker(13, seed=6)
    if name == "grid":
        return synth.grid(40, 37, seed=2)
    # odd N and isolated vertices / small components, duplicates and self-loops
    rng = np.random.default_rng(3)
    n = 1001
    e = rng.integers(0, 700, (2500, 2)).astype(np.uint32)
    e = np.concatenate([e, e[:300], np.stack([np.arange(50), np.arange(50)], 1).astype(np.uint32)])
    return e[:, 0].copy(), e[:, 1].copy(), n


@pytest.mark.parametrize("world,graph", [(2, "kron"), (3, "kron"), (2, "grid"), (3, "rand"), (1, "kron"),
                                         (4, "rand")])
def test_dist_matches_oracle(world, graph):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, graph, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
    for r, v in res.items():
        assert not isinstance(v, str), f"rank {r}: {v}"
    src, dst, n = _graph(graph)
    g = oracle.build_csr(n, src, dst)
    ro = oracle.reorder(g)
    for root, mi, lv, pa, strat, fv, fe, unv, m, nl_run, arcs in res[0]:
        ref, _, nl = oracle.bfs(g, root)
        assert arcs == g.arcs
        assert np.array_equal(lv, ref), (root, MODES[mi])
        assert oracle.validate(g, src, dst, root, lv, pa) == 0, (root, MODES[mi])
        want, _ = oracle.first_parents(ro, ref, root)
        st = np.asarray(strat + [-1])
        bu = (ref >= 1) & (st[np.clip(ref - 1, 0, len(strat))] == 2)
        assert np.array_equal(pa[bu], want[bu]), (root, MODES[mi])
        fs, fe_o = oracle.level_stats(g, ref)
        assert nl_run == nl and fv == fs.tolist() and fe == fe_o.tolist()
        assert m == oracle.input_edges(src, ref)
        opt = {k: MODES[mi][k] for k in ("alpha", "bu_stay") if k in MODES[mi]}
        if "force_strategy" in MODES[mi]:
            assert set(strat) == {MODES[mi]["force_strategy"]}
        else:
            from paper_conf_sc_yangls0w24_b200 import xbfs
            d = xbfs.xbfs_run_opts_default()
            kw = dict(alpha=d.alpha, grow=d.grow, ratio_min=d.ratio_min, bu_stay=d.bu_stay)
            kw.update(opt)
            want_s, want_u = oracle.select_sequence(g, ref, **kw)
            assert strat == want_s.tolist() and unv == want_u.tolist(), (root, MODES[mi])

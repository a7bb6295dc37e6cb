"""Host-side logic of the multi-GPU path on CPU: world_size 2 and 3 with the
gloo backend.  The real level driver (paper_conf_sc_yangls0w24_b200.dist.drive)
runs against a numpy stand-in of the per-rank device step that follows the
same partition and exchange protocol (owned rows, replicated frontier,
inbox at the owner, counters all-reduced); levels must equal the oracle's and
every rank must take the same per-level strategy."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_sc_yangls0w24_b200 import synth

BU = 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class FakeBackend:
    """numpy per-rank step with the protocol of include/xbfs_dist.h."""

    def __init__(self, g, rank, world, force=-1, alpha=0.1):
        from paper_conf_sc_yangls0w24_b200.dist import partition
        self.g, self.rank, self.world = g, rank, world
        self.n = g.n
        self.lo, self.count = partition(g.n, world, rank)
        self.force, self.alpha = force, alpha
        self.deg = g.degree()

    def _owned(self, v):
        return self.lo <= v < self.lo + self.count

    def begin(self, s, level, parent, opts):
        self.lv = level
        self.pa = parent
        self.lv[:] = -1
        self.pa[:] = -1
        self.cur = np.zeros(self.n, bool)
        self.cur[s] = True
        self.vis = np.zeros(self.n, bool)   # only the owned range is meaningful
        self.vis[s] = True
        self.k = 0
        self.log = []
        self._started = False
        owner = self._owned(s)
        if owner:
            self.lv[s - self.lo] = 0
            self.pa[s - self.lo] = s
        c = np.zeros(8, np.int64)
        c[0] = int(owner)
        c[1] = int(self.deg[s]) if owner else 0
        c[3] = int((self.deg[self.lo:self.lo + self.count] > 0).sum())
        c[4] = int(self.deg[self.lo:self.lo + self.count].sum())
        return c

    def _publish(self, owned_next):
        parts = [torch.zeros(self.n, dtype=torch.bool) for _ in range(self.world)]
        dist.all_gather(parts, torch.from_numpy(owned_next))
        return np.logical_or.reduce([p.numpy() for p in parts])

    def level(self, phase):
        g, lo, hi = self.g, self.lo, self.lo + self.count
        c = np.zeros(8, np.int64)
        if self.strategy == BU:
            nxt = np.zeros(self.n, bool)
            for v in range(lo, hi):
                if self.vis[v] or self.deg[v] == 0:
                    continue
                for u in g.col[g.row_ptr[v]:g.row_ptr[v + 1]]:
                    if self.cur[u]:
                        self.lv[v - lo] = self.k + 1
                        self.pa[v - lo] = u
                        nxt[v] = True
                        break
            self.vis |= nxt
            self.cur = self._publish(nxt)
        elif phase == 0:
            self.inbox_out = np.zeros(self.n, bool)
            self.local_next = np.zeros(self.n, bool)
            for u in np.flatnonzero(self.cur[lo:hi]) + lo:
                for v in g.col[g.row_ptr[u]:g.row_ptr[u + 1]]:
                    if self._owned(v):
                        if not self.vis[v]:
                            self.vis[v] = True
                            self.lv[v - lo] = self.k + 1
                            self.pa[v - lo] = u
                            self.local_next[v] = True
                    else:
                        self.inbox_out[v] = True
            return c
        else:
            parts = [torch.zeros(self.n, dtype=torch.bool) for _ in range(self.world)]
            dist.all_gather(parts, torch.from_numpy(self.inbox_out))   # peers' REDs into my inbox
            inbox = np.logical_or.reduce([p.numpy() for p in parts])
            nxt = self.local_next.copy()
            for v in np.flatnonzero(inbox[lo:hi]) + lo:
                if self.vis[v]:
                    continue
                for u in g.col[g.row_ptr[v]:g.row_ptr[v + 1]]:
                    if self.cur[u]:
                        self.lv[v - lo] = self.k + 1
                        self.pa[v - lo] = u
                        break
                self.vis[v] = True
                nxt[v] = True
            self.cur = self._publish(nxt)
        owned = np.flatnonzero(self.cur[lo:hi]) + lo
        c[0] = len(owned)
        c[1] = int(self.deg[owned].sum())
        return c

    def advance(self, gc):
        if not self._started:
            self._started = True
            self.fsize, self.fedges, self.arcs = int(gc[0]), int(gc[1]), int(gc[4])
        else:
            self.log.append((self.strategy, self.fsize, self.fedges))
            self.fsize, self.fedges = int(gc[0]), int(gc[1])
            self.k += 1
        self.strategy = self.force if self.force >= 0 else (BU if self.fedges > self.alpha * self.arcs else 0)
        return self.strategy, self.fsize == 0

    def levels(self):
        return self.log


def _worker(rank, world, port, scale, force, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_yangls0w24_b200.dist import drive
        src, dst, n = synth.kronecker(scale, seed=4)
        g = oracle.build_csr(n, src, dst)
        be = FakeBackend(g, rank, world, force=force, alpha=0.05)
        out = []
        for root in synth.roots(n, src, dst, 3, root_seed=7):
            level = np.empty(be.count, np.int32)
            parent = np.empty(be.count, np.int32)
            log = drive(be, lambda c: _allreduce(c), dist.barrier, int(root), level, parent, None)
            lv = [None] * world
            pa = [None] * world
            dist.all_gather_object(lv, level)
            dist.all_gather_object(pa, parent)
            out.append((int(root), np.concatenate(lv), np.concatenate(pa), [s for s, _, _ in log]))
        q.put((rank, out))
    except Exception as e:  # surface worker failures immediately
        q.put((rank, f"{type(e).__name__}: {e}"))
        raise
    finally:
        dist.destroy_process_group()


def _allreduce(c):
    t = torch.as_tensor(np.asarray(c, dtype=np.int64))
    dist.all_reduce(t)
    return t.numpy()


@pytest.mark.parametrize("world,force", [(2, -1), (3, -1), (2, 0), (2, BU)])
def test_dist_driver_gloo(world, force):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, 9, force, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=240) for _ in range(world))
    for r, v in res.items():
        assert not isinstance(v, str), f"rank {r}: {v}"
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    src, dst, n = synth.kronecker(9, seed=4)
    g = oracle.build_csr(n, src, dst)
    for i, (root, lv, pa, strat) in enumerate(res[0]):
        ref, _, nl = oracle.bfs(g, root)
        assert np.array_equal(lv, ref)
        assert oracle.validate(g, src, dst, root, lv, pa) == 0
        assert len(strat) == nl
        for r in range(1, world):                  # every rank took the same decisions
            assert res[r][i][3] == strat and np.array_equal(res[r][i][1], lv)
        if force >= 0:
            assert set(strat) == {force}


def test_partition_covers_range():
    from paper_conf_sc_yangls0w24_b200.dist import partition
    for n in (1, 31, 32, 33, 1000, 1 << 20):
        for p in (1, 2, 3, 8):
            parts = [partition(n, p, r) for r in range(p)]
            assert sum(c for _, c in parts) == n
            pos = 0
            for lo, c in parts:
                if c:
                    assert lo == pos and lo % 32 == 0
                pos += c

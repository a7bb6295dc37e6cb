"""Host-side logic of the multi-GPU path on CPU (no GPU needed): the
communicator of include/xbfs_dist.h (reading R-10: a node-local shared-memory
segment, the analogue of an NCCL communicator for the host collectives) across
world_size 2 and 3 processes, with the unique id broadcast over torch.distributed
gloo exactly as the library's users do; the partition and tuple-range rules; and
bench.py's own launcher starting 2 ranks (torch.distributed.run, 127.0.0.1)."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_sc_yangls0w24_b200.dist import Comm
        c = Comm.from_torch()
        out = []
        for it in range(200):                      # many collectives back to back (slot reuse)
            v = np.array([rank + 1, it, (rank + 1) * it, -rank], np.int64)
            out.append(c.allreduce(v).tolist())
            if it % 7 == 0:
                c.barrier()
        big = c.allreduce(np.arange(512, dtype=np.int64) * (rank + 1))
        out.append(big[:4].tolist() + [int(big[-1])])
        c.close()
        q.put((rank, out))
    except Exception as e:
        import traceback
        q.put((rank, f"{type(e).__name__}: {e}\n{traceback.format_exc()}"))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_comm_collectives_across_processes(world):
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    for r, v in res.items():
        assert not isinstance(v, str), f"rank {r}: {v}"
    s1 = world * (world + 1) // 2                   # sum of rank + 1
    for it in range(200):
        want = [s1, world * it, s1 * it, -(world * (world - 1) // 2)]
        for r in range(world):
            assert res[r][it] == want, (r, it)
    for r in range(world):
        assert res[r][200] == [0, s1, 2 * s1, 3 * s1, 511 * s1]


def test_partition_and_tuple_ranges_cover_everything():
    from paper_conf_sc_yangls0w24_b200.dist import partition, tuple_range
    for n in (1, 31, 32, 33, 1000, 1 << 20):
        for p in (1, 2, 3, 8):
            parts = [partition(n, p, r) for r in range(p)]
            assert sum(c for _, c in parts) == n
            assert all(lo % 32 == 0 for lo, c in parts if c)     # whole bitmap words per rank
            nxt = 0
            for lo, c in parts:
                if c:
                    assert lo == nxt
                    nxt = lo + c
            rngs = [tuple_range(16 * n, p, r) for r in range(p)]
            assert rngs[0][0] == 0 and rngs[-1][1] == 16 * n
            assert all(rngs[i][1] == rngs[i + 1][0] for i in range(p - 1))


def test_bench_launcher_spawns_ranks():
    """`python bench.py --gpus 2` starts 2 ranks itself (torch.distributed.run on
    127.0.0.1) when WORLD_SIZE is unset; --launcher-selftest makes every rank join
    a gloo group and the library communicator, and rank 0 print one JSON line."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--launcher-selftest"],
                       capture_output=True, text=True, timeout=300, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    d = json.loads(lines[0])
    assert d["n_ranks"] == 2 and d["allreduce"] == [3, 2] and sorted(d["ranks"]) == [0, 1]

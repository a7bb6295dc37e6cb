#!/usr/bin/env python
"""XBFS on B200 — headline benchmark (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config s24] [--impl ours|reference]

Metric: GTEPS per B200 on a Graph500 Kronecker graph (edgefactor 16), Graph500
convention (m = input tuples of the reached component, O-6), harmonic mean over
the timed roots.  A "step" is one complete BFS (init + every level) from one
root; W untimed warm-up roots precede K timed roots.  Every timed BFS is
preceded by an L2 flush (512 MiB write, outside the timed region).  Device
time per BFS = CUDA events on the library stream around init .. last level.

At N > 1 (torchrun, one process per GPU) every rank holds the same graph and
runs its own K roots (independent problems: weak scaling, no data-path
collective); value = N x min over ranks of the per-rank harmonic mean.

--impl reference times the CPU oracle (oracle/, serial FIFO BFS, 1 thread) on
the same graph and roots: the reference arm of this paper-only tier.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "GTEPS per B200 (Graph500 Kronecker, harmonic mean over 64 roots) at 1/2/4/8 GPU"

CONFIGS = {
    "s10": dict(kind="kron", scale=10, edgefactor=16),
    "s16": dict(kind="kron", scale=16, edgefactor=16),
    "s20": dict(kind="kron", scale=20, edgefactor=16),
    "s22": dict(kind="kron", scale=22, edgefactor=16),
    "s24": dict(kind="kron", scale=24, edgefactor=16),
    "s25": dict(kind="kron", scale=25, edgefactor=16),
    "s27": dict(kind="kron", scale=27, edgefactor=16),   # BASELINE config 4's graph (p = 1 point)
    "grid": dict(kind="grid", width=4096, height=4096),
    # SURVEY f4 / reading R-9: the same Kronecker tuples taken as arcs i -> j (directed BFS)
    "s24d": dict(kind="kron", scale=24, edgefactor=16, directed=True),
}
GRAPH_SEED, ROOT_SEED = 1, 2


def workload_name(cfg_name: str) -> str:
    c = CONFIGS[cfg_name]
    if c["kind"] == "kron":
        return f"graph500-kronecker-s{c['scale']}-ef{c['edgefactor']}" + ("-directed" if c.get("directed") else "")
    return f"grid-{c['width']}x{c['height']}"


def make_graph(cfg_name: str, pinned: bool):
    from paper_conf_sc_yangls0w24_b200 import synth
    c = CONFIGS[cfg_name]
    if c["kind"] == "kron":
        return synth.kronecker(c["scale"], c["edgefactor"], seed=GRAPH_SEED, pinned=pinned)
    src, dst, n = synth.grid(c["width"], c["height"], seed=GRAPH_SEED)
    return src, dst, n


def pick_roots(cfg_name: str, n, src, dst, count: int):
    from paper_conf_sc_yangls0w24_b200 import synth
    c = CONFIGS[cfg_name]
    if c["kind"] == "grid":
        W, H = c["width"], c["height"]
        fixed = [0, (H // 2) * W + W // 2]
        rnd = synth.roots(n, src, dst, count + 2, root_seed=ROOT_SEED).tolist()
        out = fixed + [r for r in rnd if r not in fixed]
        return np.array(out[:count], dtype=np.int64)
    return synth.roots(n, src, dst, count, root_seed=ROOT_SEED)


def rle(s: str) -> str:
    """Run-length form of a per-level strategy string (F=SF, S=SS, B=BU) when long."""
    if len(s) <= 24:
        return s
    out, i = [], 0
    while i < len(s):
        j = i
        while j < len(s) and s[j] == s[i]:
            j += 1
        out.append(f"{s[i]}{j - i}")
        i = j
    return " ".join(out)


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    except Exception:
        return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


def default_alpha() -> float:
    from paper_conf_sc_yangls0w24_b200.xbfs import xbfs_run_opts_default
    return xbfs_run_opts_default().alpha


def load_traffic(cfg_name: str, kernel: str):
    """DRAM bytes per launch (dram__bytes_read.sum + dram__bytes_write.sum) of
    `kernel` from the committed `ncu --set full` capture of this bench command
    (profiles/traffic.json, written by tools/ncu_traffic.py), or None."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "traffic.json")))
        return d[workload_name(cfg_name)][kernel]["dram_bytes_per_launch"]
    except Exception:
        return None


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled during the timed region."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "100"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self._t = threading.Thread(target=self._read, daemon=True)
            self._t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if not self.proc:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except Exception:
            self.proc.kill()
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx.append(float(parts[1]))
            except ValueError:
                continue
            for nm, val in zip(names, parts[3:7]):
                if val.lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


def kernel_bytes(name: str, level: int, st, n: int) -> int:
    """Algorithmic bytes of one launch, from the run's per-level counters."""
    from paper_conf_sc_yangls0w24_b200 import metrics
    if name == "init_fill":
        return metrics.bytes_init(n)
    if level < 0 or level >= st.num_levels:
        return 0
    fv, fe = st.frontier_vertices[level], st.frontier_edges[level]
    found = st.frontier_vertices[level + 1] if level + 1 < st.num_levels else 0
    if name == "td_expand_sf":
        return metrics.bytes_td_sf(n, fv, fe, found)
    if name == "td_expand_ss":
        return metrics.bytes_td_ss(n, fv, fe, found)
    if name == "generate_pre":
        return metrics.bytes_generate(n, fv, post=False)
    if name == "generate_post":
        return metrics.bytes_generate(n, found, post=True)
    if name == "ss_count":
        return metrics.bytes_ss_count(n, found)
    if name == "bu_traverse":
        return metrics.bytes_bu(n, st.unvisited[level], st.bu_probes[level], found)
    return 0


def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_yangls0w24_b200 import metrics
    from paper_conf_sc_yangls0w24_b200.xbfs import Graph

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device(f"cuda:{local}"))
    torch.cuda.set_device(local)
    dev = torch.device(f"cuda:{local}")
    t0 = time.time()
    src, dst, n = make_graph(args.config, pinned=True)
    t_gen = time.time() - t0
    total_roots = args.warmup + args.steps * world
    roots = pick_roots(args.config, n, src, dst, total_roots)
    if len(roots) < total_roots:
        roots = np.resize(roots, total_roots)
    warm = roots[: args.warmup]
    mine = roots[args.warmup + rank * args.steps: args.warmup + (rank + 1) * args.steps]

    stream = torch.cuda.current_stream(dev)
    t0 = time.time()
    directed = bool(CONFIGS[args.config].get("directed"))
    g = Graph(torch.from_numpy(src.view(np.int32)), torch.from_numpy(dst.view(np.int32)), n, device=local,
              stream=stream.cuda_stream, reorder=False, directed=directed)
    torch.cuda.synchronize()
    t_build = time.time() - t0
    t0 = time.time()
    g.reorder(1)
    torch.cuda.synchronize()
    t_reorder = time.time() - t0
    root_rule = "Graph500 (seeded, touching a non-self-loop tuple)"
    if directed:
        # R-9 root recipe: seeded candidates whose forward reach is >= 1 % of N (the giant
        # out-component; a root whose out-arcs lead to a sink reaches a handful of vertices),
        # screened with untimed runs of this library
        cand = pick_roots(args.config, n, src, dst, 4 * total_roots)
        keep = [int(r) for r in cand if g.run(int(r), stats=True)[2].vertices_reached >= n // 100]
        roots = np.resize(np.asarray(keep, dtype=np.int64), total_roots)
        warm = roots[: args.warmup]
        mine = roots[args.warmup + rank * args.steps: args.warmup + (rank + 1) * args.steps]
        root_rule = f"directed: seeded candidates with forward reach >= N/100 ({len(keep)} of {len(cand)} kept)"
        args.profile_roots = 0       # per-launch profiling runs the host-loop driver (undirected only)
    level = torch.empty(n, dtype=torch.int32, device=dev)
    parent = torch.empty(n, dtype=torch.int32, device=dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    opts = dict(driver=args.driver)
    if args.alpha is not None:
        opts["alpha"] = args.alpha
    if args.bu_stay is not None:
        opts["bu_stay"] = args.bu_stay
    if args.small_edges is not None:
        opts["small_edges"] = args.small_edges

    for r in warm:
        g.run(int(r), level, parent, stats=True, **opts)
    torch.cuda.synchronize()

    clocks = ClockSampler(local)
    clocks.start()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    per_root = []
    launches = 0
    alg_bytes = 0
    km_bytes = 0
    phase = {}          # strategy -> [levels, ms, algorithmic bytes] (persistent driver's level stamps)
    for r in mine:
        flush.fill_(1)                       # L2 flush, outside the timed region
        _, _, st = g.run(int(r), level, parent, stats=True, **opts)
        per_root.append((int(r), st.elapsed_ms, st.input_edges_traversed, st.arcs_traversed, st.num_levels,
                         "".join("FSB"[s] for s in st.strategy)))
        launches += st.kernel_launches
        lb = metrics.d3_level_bytes(n, st.strategy, st.frontier_vertices, st.frontier_edges, st.unvisited,
                                    st.bu_probes)
        alg_bytes += metrics.d3_init(n) + sum(lb)
        km_bytes += metrics.kernel_model_bytes(n, st.strategy, st.frontier_vertices, st.frontier_edges,
                                               st.unvisited, st.bu_probes, directed=directed)
        for s_, ms_, b_ in zip(st.strategy, st.level_ms, lb):
            ph = phase.setdefault("FSB"[s_], [0, 0.0, 0])
            ph[0] += 1
            ph[1] += ms_
            ph[2] += b_
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()

    teps = [m / (ms * 1e-3) for (_, ms, m, _, _, _) in per_root]
    teps_arcs = [a / (ms * 1e-3) for (_, ms, _, a, _, _) in per_root]
    hmean = metrics.harmonic_mean(teps)
    ms_mean = statistics.mean(ms for (_, ms, *_rest) in per_root)

    # parity spot check of the last timed root against a fresh run's invariants is in tests;
    # here: the parent tree of the last timed root must be consistent (cheap device check)
    lv = level.cpu().numpy()
    pa = parent.cpu().numpy()
    r_last = per_root[-1][0]
    ok_root = lv[r_last] == 0 and pa[r_last] == r_last
    reached = lv >= 0
    ok_tree = bool(ok_root and np.all(lv[pa[reached & (np.arange(n) != r_last)]] ==
                                      lv[reached & (np.arange(n) != r_last)] - 1))

    # e2e: public C-ABI call with HOST output buffers (D2H of level+parent inside)
    lh = torch.empty(n, dtype=torch.int32, pin_memory=True).numpy()
    ph = torch.empty(n, dtype=torch.int32, pin_memory=True).numpy()
    e2e_t = []
    if args.e2e_roots:
        g.run_host(int(warm[0]), lh, ph, **opts)      # warm-up: instantiates the device loop for these buffers
    for r in mine[: min(len(mine), args.e2e_roots)]:
        flush.fill_(1)
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        g.run_host(int(r), lh, ph, **opts)
        e2e_t.append(time.perf_counter() - t1)
    m_of = {r: m for (r, _, m, *_rest) in per_root}
    e2e_single = [m_of[int(r)] / t for r, t in zip(mine, e2e_t)]
    # e2e, pipelined: xbfs_run_host_batch over the same roots (D2H of root i overlaps the BFS of
    # root i+1); every root's level+parent lands in its own pinned host slot
    e2e_teps = e2e_single
    e2e_batch_s = None
    kb = min(len(mine), args.e2e_roots)
    if kb >= 2:
        lhb = torch.empty(kb * n, dtype=torch.int32, pin_memory=True).numpy()
        phb = torch.empty(kb * n, dtype=torch.int32, pin_memory=True).numpy()
        g.run_host_batch(np.asarray(warm[:2], dtype=np.int64), lhb, phb, **opts)   # warm-up
        roots_b = np.asarray(mine[:kb], dtype=np.int64)
        flush.fill_(1)
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        g.run_host_batch(roots_b, lhb, phb, **opts)
        e2e_batch_s = time.perf_counter() - t1
        e2e_teps = [m_of[int(r)] / (e2e_batch_s / kb) for r in roots_b]
        # the host copy is the result: check the last root's tree against the device run's levels
        lb = lhb[(kb - 1) * n:kb * n]
        assert lb[int(roots_b[-1])] == 0 and phb[(kb - 1) * n + int(roots_b[-1])] == int(roots_b[-1])

    # roofline: per-launch event timing of a few roots (host-loop driver)
    peak, peak_src = load_peaks()
    agg = {}
    for r in mine[: min(len(mine), args.profile_roots)]:
        flush.fill_(1)
        _, _, st = g.run(int(r), level, parent, stats=True, profile=8192, driver=1)
        for (name, lvl, ms) in st.kernels:
            b = kernel_bytes(name, lvl, st, n)
            a = agg.setdefault(name, [0, 0.0, 0])
            a[0] += 1
            a[1] += ms
            a[2] += b
    kernels = {k: {"launches": v[0], "total_ms": round(v[1], 4), "avg_ms": round(v[1] / v[0], 5),
                   "bytes_per_launch": int(v[2] / v[0]),
                   "gbs": round(v[2] / (v[1] * 1e-3) / 1e9, 1) if v[1] > 0 else None}
               for k, v in agg.items()}
    roofline = None
    timed_ms = sum(x[1] for x in per_root)
    if launches == len(per_root):
        # persistent driver: the timed region is ONE kernel launch per BFS (k_persist),
        # so its event time per BFS is that kernel's launch duration
        ach = alg_bytes / (timed_ms * 1e-3) / 1e9
        bpl = int(alg_bytes / len(per_root))
        roofline = {"bound": "hbm", "kernel": "k_persist", "achieved": round(ach, 1), "peak": peak, "unit": "GB/s",
                    "frac": round(ach / peak, 4), "traffic": load_traffic(args.config, "k_persist"),
                    "bytes_per_launch": bpl, "launch_ms": round(timed_ms / len(per_root), 4),
                    "peak_source": peak_src,
                    "phases": {k: {"levels": v[0], "ms": round(v[1], 4),
                                   "gbs": round(v[2] / (v[1] * 1e-3) / 1e9, 1) if v[1] > 0 else None}
                               for k, v in phase.items()},
                    "kernel_model": {"bytes_per_launch": int(km_bytes / len(per_root)),
                                     "gbs": round(km_bytes / (timed_ms * 1e-3) / 1e9, 1),
                                     "note": "what this build's kernels move by their own traffic model "
                                             "(metrics.kernel_model_bytes); context, not the numerator"},
                    "note": "achieved = SURVEY §8(d) D-3 algorithmic bytes (init + every level, replayed by "
                            "oracle_byte_replay) / event time of the single k_persist launch per BFS, over the "
                            "timed roots; phases from the kernel's %globaltimer level stamps"}
    elif agg:
        dom = max(agg.items(), key=lambda kv: kv[1][1])[0]
        d = kernels[dom]
        ach = d["gbs"]
        roofline = {"bound": "hbm", "kernel": dom, "achieved": ach, "peak": peak, "unit": "GB/s",
                    "frac": round(ach / peak, 4) if ach else None, "traffic": load_traffic(args.config, dom),
                    "bytes_per_launch": d["bytes_per_launch"], "peak_source": peak_src}
    b_model = metrics.model_bytes(n, g.arcs)
    model_frac = b_model / (ms_mean * 1e-3) / (peak * 1e9)

    res = dict(rank=rank, hmean=hmean, per_root=per_root, launches=launches, ms_mean=ms_mean,
               e2e=metrics.harmonic_mean(e2e_teps) if e2e_teps else None,
               e2e_single=metrics.harmonic_mean(e2e_single) if e2e_single else None,
               e2e_batch_roots=kb if e2e_batch_s is not None else 0, clocks=clk, ok_tree=ok_tree,
               roofline=roofline, kernels=kernels, teps_arcs=metrics.harmonic_mean(teps_arcs),
               model_frac=model_frac, quart=metrics.quartiles(teps))
    if world > 1:
        allres = [None] * world
        dist.all_gather_object(allres, res)
    else:
        allres = [res]
    if rank != 0:
        g.close()
        if world > 1:
            dist.destroy_process_group()
        return

    worst = min(allres, key=lambda x: x["hmean"])
    value = world * worst["hmean"] / 1e9
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(args, src, dst, n, mine, m_of)
    line = {
        "metric": METRIC,
        "value": round(value, 3),
        "unit": "GTEPS",
        "n_gpus": world,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(max(x["ms_mean"] for x in allres), 4),
        "higher_is_better": True,
        "scaling": "weak",
        "vs_baseline": None,
        "dtype": "int32",
        "data": "synthetic (seeded Graph500 Kronecker generator, graph seed 1, root seed 2)",
        "config": {"workload": workload_name(args.config), "n_vertices": n, "input_edges": int(src.shape[0]),
                   "arcs": g.arcs, "roots_per_gpu": args.steps, "l2_flush": "512 MiB write before every timed BFS",
                   "reorder": "degree-desc (P:L153)", "alpha": opts.get("alpha", default_alpha()),
                   "roots": root_rule,
                   "bu_stay": opts.get("bu_stay", 1.0),
                   "driver": {0: "persistent (auto)", 1: "host loop", 2: "CUDA-graph loop",
                              3: "persistent"}[args.driver],
                   "parallelism": f"replicas x{world} (independent roots)"},
        "gteps_hmean_per_gpu": round(worst["hmean"] / 1e9, 3),
        "gteps_arcs_hmean": round(res["teps_arcs"] / 1e9, 3),
        "gteps_quartiles": {k: round(v / 1e9, 3) for k, v in res["quart"].items()},
        "roofline_model": {"bytes": b_model, "formula": "16N + 4A (P:L358)", "frac": round(model_frac, 4),
                           "peak_gbs": peak},
        "clocks": res["clocks"],
        "e2e": {"value": round(res["e2e"] / 1e9, 3) if res["e2e"] else None, "unit": "GTEPS",
                "h2d_bytes_per_step": 8, "d2h_bytes_per_step": 8 * n,
                "single_call_value": round(res["e2e_single"] / 1e9, 3) if res["e2e_single"] else None,
                "roots": res["e2e_batch_roots"],
                "note": "xbfs_run_host_batch over the first roots (one call, wall clock): source scalars in, "
                        "level+parent (int32 each) of every root D2H into its own pinned host slot, the copy "
                        "of root i overlapping the BFS of root i+1 (no L2 flush between roots inside the call; "
                        "each BFS's 134 MB output fill and the 2 GB CSR exceed L2); single_call_value = "
                        "xbfs_run_host one root per call, L2 flushed before each"},
        "gpu_launches": int(sum(x["launches"] for x in allres)),
        "roofline": res["roofline"],
        "kernels": res["kernels"],
        "cpu_baseline": cpu,
        "levels": [pr[4] for pr in res["per_root"][:4]],
        "strategies": [rle(pr[5]) for pr in res["per_root"][:4]],
        "parent_tree_consistent": bool(all(x["ok_tree"] for x in allres)),
        "prep_s": {"generate": round(t_gen, 2), "build_csr": round(t_build, 2), "reorder": round(t_reorder, 2)},
    }
    print(json.dumps(line), flush=True)
    g.close()
    if world > 1:
        dist.destroy_process_group()


def cpu_baseline(args, src, dst, n, roots, m_of=None, budget_s=None):
    """The oracle as it stands (serial FIFO BFS, 1 thread) on a bounded sample of
    the same workload: the first roots until ~budget seconds of BFS time."""
    import oracle
    budget_s = args.cpu_budget if budget_s is None else budget_s
    t0 = time.time()
    og = (oracle.build_csr_directed if CONFIGS[args.config].get("directed") else oracle.build_csr)(n, src, dst)
    t_csr = time.time() - t0
    teps, used, spent = [], [], 0.0
    for r in roots:
        t1 = time.perf_counter()
        lv, _, _ = oracle.bfs(og, int(r))
        dt = time.perf_counter() - t1
        m = oracle.input_edges(src, lv)
        teps.append(m / dt)
        used.append(int(r))
        spent += dt
        if spent >= budget_s:
            break
    from paper_conf_sc_yangls0w24_b200 import metrics
    return {"value": round(metrics.harmonic_mean(teps) / 1e9, 5), "unit": "GTEPS", "cores": 1, "kind": "oracle",
            "sample": f"{len(used)} of the timed roots of {workload_name(args.config)} (serial BFS, oracle CSR "
                      f"prebuilt in {t_csr:.1f}s untimed), {spent:.1f}s of BFS",
            "host_cores": os.cpu_count()}


def run_reference(args):
    """Reference arm: the CPU oracle timed as it stands (rank 0 only)."""
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    from paper_conf_sc_yangls0w24_b200 import metrics
    src, dst, n = make_graph(args.config, pinned=False)
    directed = bool(CONFIGS[args.config].get("directed"))
    roots = pick_roots(args.config, n, src, dst, 4 * (args.warmup + args.steps * world) if directed
                       else args.warmup + args.steps * world)
    og = (oracle.build_csr_directed if directed else oracle.build_csr)(n, src, dst)
    for r in roots[: args.warmup]:
        oracle.bfs(og, int(r))
    teps, times = [], []
    for r in roots[args.warmup:]:
        if len(teps) == args.steps:
            break
        t1 = time.perf_counter()
        lv, _, _ = oracle.bfs(og, int(r))
        dt = time.perf_counter() - t1
        if directed and int((lv >= 0).sum()) < n // 100:
            continue                 # the R-9 root rule (forward reach >= N/100), as in our arm
        teps.append(oracle.input_edges(src, lv) / dt)
        times.append(dt)
    value = metrics.harmonic_mean(teps) / 1e9
    line = {
        "impl": "reference", "metric": METRIC, "value": round(value, 5), "unit": "GTEPS", "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(1e3 * statistics.mean(times), 3),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "config": {"workload": workload_name(args.config), "n_vertices": n, "input_edges": int(src.shape[0]),
                   "arcs": og.arcs},
        "cpu_baseline": {"value": round(value, 5), "unit": "GTEPS", "cores": 1, "kind": "oracle",
                         "sample": f"{args.steps} roots, one full serial BFS each (oracle CSR prebuilt, untimed)"},
        "e2e": {"value": round(value, 5), "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=64)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="s24", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--driver", type=int, default=0,
                    help="0 auto (= 3), 1 host loop, 2 CUDA-graph device loop, 3 persistent kernel")
    ap.add_argument("--alpha", type=float, default=None)
    ap.add_argument("--bu-stay", type=float, default=None)
    ap.add_argument("--small-edges", type=int, default=None)
    ap.add_argument("--e2e-roots", type=int, default=16)
    ap.add_argument("--profile-roots", type=int, default=4)
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--mode", default="auto", choices=["auto", "dist", "replicas"],
                    help="N>1: dist = one graph 1D-partitioned over the N GPUs (default), "
                         "replicas = every GPU its own copy and roots")
    args = ap.parse_args()
    assert args.warmup >= 3 or args.impl == "reference" or os.environ.get("XBFS_ALLOW_SHORT_WARMUP"), \
        "timing rules: at least 3 warm-up steps"
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.impl == "reference":
        run_reference(args)
    elif args.mode == "dist" or (args.mode == "auto" and world > 1):
        run_dist(args)
    else:
        run_ours(args)


def run_dist(args):
    """One BFS per step over ONE graph 1D-partitioned across the N ranks
    (include/xbfs_dist.h): strong scaling of the same s24 workload.  Per-BFS
    time = max over ranks of the CUDA-event time around the rank's whole level
    loop (host collectives included); value = harmonic mean of m / t."""
    import torch
    import torch.distributed as dist

    from paper_conf_sc_yangls0w24_b200 import metrics
    from paper_conf_sc_yangls0w24_b200.dist import DistGraph

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device(f"cuda:{local}")
    if world == 1:
        for k, v in dict(RANK="0", WORLD_SIZE="1", MASTER_ADDR="127.0.0.1", MASTER_PORT="29517").items():
            os.environ.setdefault(k, v)
    dist.init_process_group("nccl" if world > 1 else "gloo", device_id=dev if world > 1 else None)
    t0 = time.time()
    src, dst, n = make_graph(args.config, pinned=True)
    t_gen = time.time() - t0
    roots = pick_roots(args.config, n, src, dst, args.warmup + args.steps)
    opts = {}
    if args.alpha is not None:
        opts["alpha"] = args.alpha
    if args.bu_stay is not None:
        opts["bu_stay"] = args.bu_stay
    t0 = time.time()
    dg = DistGraph(torch.from_numpy(src.view(np.int32)), torch.from_numpy(dst.view(np.int32)), n, device=local)
    torch.cuda.synchronize()
    t_build = time.time() - t0
    del src, dst
    level = torch.empty(max(dg.count, 1), dtype=torch.int32, device=dev)[: dg.count]
    parent = torch.empty(max(dg.count, 1), dtype=torch.int32, device=dev)[: dg.count]
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    for r in roots[: args.warmup]:
        dg.run(int(r), level, parent, **opts)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    clocks = ClockSampler(local)
    clocks.start()
    per = []
    for r in roots[args.warmup:]:
        flush.fill_(1)
        torch.cuda.synchronize()
        dist.barrier()
        ev0.record()
        _, _, st = dg.run(int(r), level, parent, **opts)
        ev1.record()
        ev1.synchronize()
        ms = torch.tensor([ev0.elapsed_time(ev1)], dtype=torch.float64, device=dev if world > 1 else "cpu")
        dist.all_reduce(ms, op=dist.ReduceOp.MAX)
        per.append((int(r), float(ms.item()), st.input_edges_traversed, sum(st.frontier_edges), st.num_levels,
                    "".join("FSB"[s] for s in st.strategy)))
    clk = clocks.stop()
    reached = torch.tensor([int((level >= 0).sum().item())], dtype=torch.int64,
                           device=dev if world > 1 else "cpu")
    dist.all_reduce(reached)
    if rank == 0:
        teps = [m / (ms * 1e-3) for (_, ms, m, _, _, _) in per]
        hm = metrics.harmonic_mean(teps)
        ms_mean = statistics.mean(ms for (_, ms, *_r) in per)
        peak, peak_src = load_peaks()
        line = {
            "metric": METRIC, "value": round(hm / 1e9, 3), "unit": "GTEPS", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_mean, 4), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic (seeded Graph500 Kronecker generator, graph seed 1, root seed 2)",
            "config": {"workload": workload_name(args.config), "n_vertices": n, "roots": args.steps,
                       "parallelism": f"1D vertex partition x{world} (xbfs_dist, peer-memory frontier exchange)",
                       "l2_flush": "512 MiB write before every timed BFS", "alpha": opts.get("alpha", default_alpha()),
                       "bu_stay": opts.get("bu_stay", 1.0)},
            "gteps_per_gpu": round(hm / 1e9 / world, 3),
            "gteps_arcs_hmean": round(metrics.harmonic_mean([a / (ms * 1e-3) for (_, ms, _, a, _, _) in per]) / 1e9,
                                      3),
            "clocks": clk,
            "e2e": None,
            "gpu_launches": None,
            "roofline": None,
            "cpu_baseline": None,
            "levels": [p[4] for p in per[:4]],
            "strategies": [rle(p[5]) for p in per[:4]],
            "reached_last_root": int(reached.item()),
            "prep_s": {"generate": round(t_gen, 2), "build_dist": round(t_build, 2)},
            "peak_gbs": peak, "peak_source": peak_src,
        }
        print(json.dumps(line), flush=True)
    dg.close()
    dist.destroy_process_group()


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""XBFS on B200 — headline benchmark (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config NAME] [--impl ours|reference]

Metric: GTEPS per B200 on a Graph500 Kronecker graph (edgefactor 16), Graph500
convention (m = input tuples of the reached component, O-6), harmonic mean over
the timed roots.  A "step" is one complete BFS (init + every level) from one
root; W untimed warm-up roots precede K timed roots.  Every timed BFS is
preceded by an L2 flush (512 MiB write, outside the timed region).  Device time
per BFS = CUDA events on the library stream; at N > 1 the max over ranks.
Every timed root is then validated on the device (Graph500 V1-V5 over all input
tuples, which certify the levels exactly) outside the timed region.

N = 1 (default config s24, BASELINE config 3): one process, the persistent
kernel, xbfs_run.  N > 1 (default config s27, BASELINE config 4): one process
per GPU — launched here with torch.distributed.run on 127.0.0.1 when WORLD_SIZE
is unset, or by the caller's torchrun — every rank generates only its share of
the tuples, xbfs_build_csr_dist partitions the graph 1D by vertex, and one
xbfs_run_dist call per BFS runs it on all GPUs (strong scaling of one graph);
value = total GTEPS / N (per B200, as the metric names it), gteps_total beside it.

--impl reference times the CPU oracle (oracle/, serial FIFO BFS, 1 thread) on
the same graph and roots: the reference arm of this paper-only tier.
"""
from __future__ import annotations

import argparse
import json
import os
import socket
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
    "s27": dict(kind="kron", scale=27, edgefactor=16),   # BASELINE config 4's graph
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


def make_graph(cfg_name: str, pinned: bool, e_range=None):
    """(src, dst, n) of the whole workload, or of tuples [e0, e1) when e_range is given."""
    from paper_conf_sc_yangls0w24_b200 import synth
    c = CONFIGS[cfg_name]
    if c["kind"] == "kron":
        e0, e1 = e_range if e_range else (0, None)
        return synth.kronecker(c["scale"], c["edgefactor"], seed=GRAPH_SEED, pinned=pinned, e_begin=e0, e_end=e1)
    src, dst, n = synth.grid(c["width"], c["height"], seed=GRAPH_SEED)
    if e_range:
        src, dst = src[e_range[0]:e_range[1]].copy(), dst[e_range[0]:e_range[1]].copy()
    return src, dst, n


def num_tuples(cfg_name: str) -> int:
    c = CONFIGS[cfg_name]
    if c["kind"] == "kron":
        return c["edgefactor"] << c["scale"]
    from paper_conf_sc_yangls0w24_b200 import synth
    return int(synth.lib().synth_grid_count(c["width"], c["height"]))


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


def pick_roots_dist(comm, n, src_local, dst_local, count: int):
    """O-7 roots when every rank holds only its share of the tuples: the same
    candidate stream as synth.roots (splitmix64(root_seed + t) mod N, repeats
    skipped), a candidate eligible iff some rank's share has a non-self-loop
    tuple touching it (flags summed over the library communicator)."""
    from paper_conf_sc_yangls0w24_b200 import synth
    nz = src_local != dst_local
    s_nz, d_nz = src_local[nz], dst_local[nz]
    out, seen, t = [], set(), 0
    while len(out) < count:
        cand = []
        while len(cand) < max(64, 4 * (count - len(out))):
            v = synth.splitmix64(ROOT_SEED + t) % n
            t += 1
            if v not in seen:
                seen.add(v)
                cand.append(v)
        ci = np.asarray(cand, dtype=np.int64)
        tbl = np.zeros(n, dtype=bool)
        tbl[ci] = True
        hit = np.zeros(n, dtype=bool)
        hit[s_nz[tbl[s_nz]]] = True
        hit[d_nz[tbl[d_nz]]] = True
        flags = comm.allreduce(hit[ci].astype(np.int64))
        out += [v for v, f in zip(cand, flags) if f > 0]
    return np.asarray(out[:count], dtype=np.int64)


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


def bench_config(args, n: int, m: int, arcs: int, world: int) -> dict:
    """The config dict, identical for our arm and the reference arm."""
    return {"workload": workload_name(args.config), "n_vertices": int(n), "input_edges": int(m), "arcs": int(arcs),
            "roots": args.steps, "l2_flush": "512 MiB write before every timed BFS (inputs > L2)",
            "reorder": "degree-desc (P:L153)", "alpha": args.alpha if args.alpha is not None else default_alpha(),
            "bu_stay": args.bu_stay if args.bu_stay is not None else 1.0,
            "parallelism": ("1 GPU" if world == 1 else
                            f"1D vertex partition x{world} (xbfs_run_dist, peer-memory frontier exchange)")}


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


# ---------------------------------------------------------------------------
# Graph500 validation of a timed root on the device (harness check, untimed):
# V1 root, V2 reached <=> parent (unreached: exactly -1/-1), V3 level step,
# V4 tree edge is an input tuple, V5 every tuple spans <= 1 level (both or
# neither endpoint reached).  V1-V5 pin the levels exactly.
# ---------------------------------------------------------------------------

def _validate_tuples(src, dst, level, parent, ok, directed, chunk=1 << 26):
    """V5 over this process's tuples; marks ok[v] where (parent[v], v) is a tuple."""
    bad = 0
    for e0 in range(0, src.shape[0], chunk):
        i = src[e0:e0 + chunk].long()
        j = dst[e0:e0 + chunk].long()
        li, lj = level[i], level[j]
        nl = i != j
        if directed:
            if bool(((li >= 0) & nl & ((lj < 0) | (lj > li + 1))).any()):
                bad |= 16
            sel = nl & (lj >= 0) & (parent[j].long() == i)
            ok[j[sel]] = True
        else:
            if bool(((li >= 0) != (lj >= 0)).any()) or bool(((li >= 0) & ((li - lj).abs() > 1)).any()):
                bad |= 16
            sel = nl & (li >= 0)
            ok[j[sel & (parent[j].long() == i)]] = True
            ok[i[sel & (parent[i].long() == j)]] = True
        del i, j, li, lj, nl
    return bad


def _validate_vertices(n, root, level, parent):
    bad = 0
    if int(parent[root]) != root or int(level[root]) != 0:
        bad |= 1
    reached = level >= 0
    if bool((reached != (parent >= 0)).any()) or bool(((~reached) & ((level != -1) | (parent != -1))).any()):
        bad |= 2
    v = reached.clone()
    v[root] = False
    pv = parent[v].long()
    if bool((pv >= n).any()):
        return bad | 32
    if bool((level[pv] != level[v] - 1).any()):
        bad |= 4
    return bad


def gpu_validate(src_d, dst_d, n, root, level, parent, directed=False):
    """0 iff the (device) level/parent pass V1-V5 against the (device) tuples."""
    import torch
    bad = _validate_vertices(n, root, level, parent)
    if bad & 32:
        return bad
    ok = torch.zeros(n, dtype=torch.bool, device=level.device)
    bad |= _validate_tuples(src_d, dst_d, level, parent, ok, directed)
    need = level >= 0
    need[root] = False
    if bool((need & ~ok).any()):
        bad |= 8
    return bad


# ---------------------------------------------------------------------------
# N = 1: the persistent kernel through xbfs_run
# ---------------------------------------------------------------------------

def run_ours(args):
    import torch

    from paper_conf_sc_yangls0w24_b200 import metrics
    from paper_conf_sc_yangls0w24_b200.xbfs import Graph

    torch.cuda.set_device(0)
    dev = torch.device("cuda:0")
    t0 = time.time()
    src, dst, n = make_graph(args.config, pinned=True)
    t_gen = time.time() - t0
    total_roots = args.warmup + args.steps
    roots = pick_roots(args.config, n, src, dst, total_roots)
    if len(roots) < total_roots:
        roots = np.resize(roots, total_roots)
    warm = roots[: args.warmup]
    mine = roots[args.warmup: args.warmup + args.steps]

    stream = torch.cuda.current_stream(dev)
    t0 = time.time()
    directed = bool(CONFIGS[args.config].get("directed"))
    src_d = torch.from_numpy(src.view(np.int32)).to(dev)
    dst_d = torch.from_numpy(dst.view(np.int32)).to(dev)
    g = Graph(src_d, dst_d, n, device=0, stream=stream.cuda_stream, reorder=False, directed=directed)
    torch.cuda.synchronize()
    t_build = time.time() - t0
    t0 = time.time()
    g.reorder(1)
    torch.cuda.synchronize()
    t_reorder = time.time() - t0
    root_rule = "Graph500 (seeded, touching a non-self-loop tuple)"
    reach = None
    if directed:
        # R-9 root recipe: seeded candidates whose forward reach is >= 1 % of N (the giant
        # out-component; a root whose out-arcs lead to a sink reaches a handful of vertices),
        # screened with untimed runs of this library.  This biases the mean up against
        # unscreened seeded roots; both are reported.
        cand = pick_roots(args.config, n, src, dst, 4 * total_roots)
        reach = {int(r): g.run(int(r), stats=True)[2] for r in cand}
        keep = [r for r in reach if reach[r].vertices_reached >= n // 100]
        if not keep:
            raise SystemExit("s24d: no seeded root reaches N/100 vertices")
        roots = np.resize(np.asarray(keep, dtype=np.int64), total_roots)
        warm = roots[: args.warmup]
        mine = roots[args.warmup: args.warmup + args.steps]
        root_rule = f"directed: seeded candidates with forward reach >= N/100 ({len(keep)} of {len(cand)} kept)"
        args.profile_roots = 0       # per-launch profiling runs the host-loop driver (undirected only)
    level = torch.empty(n, dtype=torch.int32, device=dev)
    parent = torch.empty(n, dtype=torch.int32, device=dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    opts = dict(driver=args.driver)
    for k in ("alpha", "bu_stay", "small_edges"):
        if getattr(args, k) is not None:
            opts[k] = getattr(args, k)

    for r in warm:
        g.run(int(r), level, parent, stats=True, **opts)
    torch.cuda.synchronize()

    clocks = ClockSampler(0)
    clocks.start()
    torch.cuda.synchronize()
    per_root, bad_roots = [], []
    launches = 0
    alg_bytes = km_bytes = 0
    init_ms = 0.0
    phase = {}          # strategy -> [levels, ms, algorithmic bytes] (persistent driver's level stamps)
    for r in mine:
        flush.fill_(1)                       # L2 flush, outside the timed region
        _, _, st = g.run(int(r), level, parent, stats=True, **opts)
        # untimed: validate this root's result on the device (V1-V5 over all tuples)
        if not args.no_validate:
            bad = gpu_validate(src_d, dst_d, n, int(r), level, parent, directed)
            if bad:
                bad_roots.append((int(r), bad))
        per_root.append((int(r), st.elapsed_ms, st.input_edges_traversed, st.arcs_traversed, st.num_levels,
                         "".join("FSB"[s] for s in st.strategy)))
        launches += st.kernel_launches
        init_ms += st.init_ms
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
    clk = clocks.stop()
    if bad_roots:
        raise SystemExit(f"validation FAILED for timed roots {bad_roots[:5]} (V-check bitmask)")

    teps = [m / (ms * 1e-3) for (_, ms, m, _, _, _) in per_root]
    teps_arcs = [a / (ms * 1e-3) for (_, ms, _, a, _, _) in per_root]
    hmean = metrics.harmonic_mean(teps)
    ms_mean = statistics.mean(ms for (_, ms, *_rest) in per_root)
    timed_ms = sum(x[1] for x in per_root)
    m_of = {r: m for (r, _, m, *_rest) in per_root}

    # e2e: public C-ABI call with HOST output buffers (D2H of level+parent inside)
    lh = torch.empty(n, dtype=torch.int32, pin_memory=True).numpy()
    ph_ = torch.empty(n, dtype=torch.int32, pin_memory=True).numpy()
    e2e_t = []
    if args.e2e_roots:
        g.run_host(int(warm[0]), lh, ph_, **opts)
    for r in mine[: min(len(mine), args.e2e_roots)]:
        flush.fill_(1)
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        g.run_host(int(r), lh, ph_, **opts)
        e2e_t.append(time.perf_counter() - t1)
    e2e_single = [m_of[int(r)] / t for r, t in zip(mine, e2e_t)]
    # e2e, pipelined: xbfs_run_host_batch over the same roots (D2H of root i overlaps the BFS of
    # root i+1); every root's level+parent lands in its own pinned host slot
    e2e_teps = e2e_single
    kb = min(len(mine), args.e2e_roots)
    e2e_batch = False
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
        e2e_batch = True
        # the host copy is the result: the last root's host levels are a tree from it
        lb_ = lhb[(kb - 1) * n:kb * n]
        assert lb_[int(roots_b[-1])] == 0 and phb[(kb - 1) * n + int(roots_b[-1])] == int(roots_b[-1])

    # per-launch event timing of a few roots (host-loop driver): shares of the step
    peak, peak_src = load_peaks()
    agg = {}
    for r in mine[: min(len(mine), args.profile_roots)]:
        flush.fill_(1)
        _, _, st = g.run(int(r), level, parent, stats=True, profile=4096, driver=1)
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
    if launches == len(per_root):
        # persistent driver: the timed region is ONE kernel launch per BFS (k_persist),
        # so its event time per BFS is that kernel's launch duration
        ach = alg_bytes / (timed_ms * 1e-3) / 1e9
        phases = {k: {"levels": v[0], "ms": round(v[1], 4),
                      "gbs": round(v[2] / (v[1] * 1e-3) / 1e9, 1) if v[1] > 0 else None}
                  for k, v in phase.items()}
        phases["init"] = {"ms": round(init_ms, 4),
                          "gbs": round(len(per_root) * metrics.d3_init(n) / (init_ms * 1e-3) / 1e9, 1)
                          if init_ms > 0 else None}
        roofline = {"bound": "hbm", "kernel": "k_persist", "achieved": round(ach, 1), "peak": peak, "unit": "GB/s",
                    "frac": round(ach / peak, 4), "traffic": load_traffic(args.config, "k_persist"),
                    "bytes_per_launch": int(alg_bytes / len(per_root)),
                    "launch_ms": round(timed_ms / len(per_root), 4), "peak_source": peak_src, "phases": phases,
                    "kernel_model": {"bytes_per_launch": int(km_bytes / len(per_root)),
                                     "gbs": round(km_bytes / (timed_ms * 1e-3) / 1e9, 1),
                                     "note": "what this build's kernels move by their own traffic model "
                                             "(metrics.kernel_model_bytes); context, not the numerator"},
                    "note": "achieved = SURVEY §8(d) D-3 algorithmic bytes (init + every level, replayed by "
                            "oracle_byte_replay) / event time of the single k_persist launch per BFS, over the "
                            "timed roots; phases from the kernel's %globaltimer stamps (ms summed over roots)"}
    b_model = metrics.model_bytes(n, g.arcs)
    model_frac = b_model / (ms_mean * 1e-3) / (peak * 1e9)

    cpu = None if args.no_cpu_baseline else cpu_baseline(args, src, dst, n, mine)
    line = {
        "metric": METRIC,
        "value": round(hmean / 1e9, 3),
        "unit": "GTEPS",
        "n_gpus": 1,
        "steps": args.steps,
        "warmup": args.warmup,
        "ms_per_step": round(ms_mean, 4),
        "higher_is_better": True,
        "scaling": "strong",
        "vs_baseline": None,
        "dtype": "int32",
        "data": "synthetic (seeded Graph500 Kronecker generator, graph seed 1, root seed 2)",
        "config": dict(bench_config(args, n, src.shape[0], g.arcs, 1), root_rule=root_rule,
                       driver={0: "persistent (auto)", 1: "host loop", 2: "CUDA-graph loop",
                               3: "persistent"}[args.driver]),
        "gteps_total": round(hmean / 1e9, 3),
        "gteps_arcs_hmean": round(metrics.harmonic_mean(teps_arcs) / 1e9, 3),
        "gteps_quartiles": {k: round(v / 1e9, 3) for k, v in metrics.quartiles(teps).items()},
        "validated_roots": f"{len(per_root) - len(bad_roots)}/{len(per_root)}" if not args.no_validate else "skipped",
        "roofline_model": {"bytes": b_model, "formula": "16N + 4A (P:L358)", "frac": round(model_frac, 4),
                           "peak_gbs": peak},
        "clocks": clk,
        "e2e": {"value": round(metrics.harmonic_mean(e2e_teps) / 1e9, 3) if e2e_teps else None, "unit": "GTEPS",
                "h2d_bytes_per_step": 8, "d2h_bytes_per_step": 8 * n,
                "single_call_value": round(metrics.harmonic_mean(e2e_single) / 1e9, 3) if e2e_single else None,
                "roots": kb if e2e_batch else len(e2e_single),
                "note": "xbfs_run_host_batch over the first roots (one call, wall clock): source scalars in, "
                        "level+parent (int32 each) of every root D2H into its own pinned host slot, the copy "
                        "of root i overlapping the BFS of root i+1; single_call_value = xbfs_run_host one root "
                        "per call, L2 flushed before each"},
        "gpu_launches": int(launches),
        "roofline": roofline,
        "kernels": kernels,
        "cpu_baseline": cpu,
        "levels": [pr[4] for pr in per_root[:4]],
        "strategies": [rle(pr[5]) for pr in per_root[:4]],
        "prep_s": {"generate": round(t_gen, 2), "build_csr": round(t_build, 2), "reorder": round(t_reorder, 2)},
    }
    if reach is not None:
        line["config"]["unscreened_roots"] = {
            "gteps_hmean": round(metrics.harmonic_mean(
                [reach[r].input_edges_traversed / (reach[r].elapsed_ms * 1e-3) for r in reach
                 if reach[r].elapsed_ms > 0 and reach[r].input_edges_traversed > 0]) / 1e9, 3),
            "note": "all seeded candidates incl. those reaching < N/100 (stats runs, no L2 flush): the screening "
                    "bias of the headline"}
    print(json.dumps(line), flush=True)
    g.close()


def kernel_bytes(name: str, level: int, st, n: int) -> int:
    """Kernel-model bytes of one launch, from the run's per-level counters."""
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


# ---------------------------------------------------------------------------
# N > 1: one graph partitioned over the ranks, xbfs_run_dist
# ---------------------------------------------------------------------------

def run_dist(args):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_yangls0w24_b200 import metrics
    from paper_conf_sc_yangls0w24_b200.dist import Comm, DistGraph, tuple_range

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device(f"cuda:{local}")
    if world == 1:
        for k, v in dict(RANK="0", WORLD_SIZE="1", MASTER_ADDR="127.0.0.1", MASTER_PORT=str(_free_port())).items():
            os.environ.setdefault(k, v)
    dist.init_process_group("nccl", device_id=dev)
    comm = Comm.from_torch()
    if CONFIGS[args.config].get("directed"):
        raise SystemExit("directed graphs are single-GPU only")
    t0 = time.time()
    m_all = num_tuples(args.config)
    e0, e1 = tuple_range(m_all, world, rank)
    src, dst, n = make_graph(args.config, pinned=True, e_range=(e0, e1))
    t_gen = time.time() - t0
    roots = pick_roots_dist(comm, n, src, dst, args.warmup + args.steps)
    opts = {k: getattr(args, k) for k in ("alpha", "bu_stay") if getattr(args, k) is not None}
    t0 = time.time()
    src_d = torch.from_numpy(src.view(np.int32)).to(dev)
    dst_d = torch.from_numpy(dst.view(np.int32)).to(dev)
    dg = DistGraph(comm, src_d, dst_d, n, device=local)
    torch.cuda.synchronize()
    t_build = time.time() - t0
    level = torch.empty(max(dg.count, 1), dtype=torch.int32, device=dev)[: dg.count]
    parent = torch.empty(max(dg.count, 1), dtype=torch.int32, device=dev)[: dg.count]
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    blk = 32 * ((n + 32 * world - 1) // (32 * world))
    full_l = torch.empty(world * blk, dtype=torch.int32, device=dev)
    full_p = torch.empty(world * blk, dtype=torch.int32, device=dev)
    pad_l = torch.full((blk,), -1, dtype=torch.int32, device=dev)
    pad_p = torch.full((blk,), -1, dtype=torch.int32, device=dev)

    def tmax(x):
        t = torch.tensor([float(x)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def validate(root):
        # the partition is rank-ordered blocks of `blk`: gather every rank's slice everywhere
        pad_l[: dg.count] = level
        pad_p[: dg.count] = parent
        dist.all_gather_into_tensor(full_l, pad_l)
        dist.all_gather_into_tensor(full_p, pad_p)
        lv, pa = full_l[:n], full_p[:n]
        ok = torch.zeros(n, dtype=torch.bool, device=dev)
        bad = _validate_tuples(src_d, dst_d, lv, pa, ok, False)
        okk = ok.to(torch.uint8)
        dist.all_reduce(okk, op=dist.ReduceOp.MAX)
        need = lv >= 0
        need[root] = False
        if bool((need & (okk == 0)).any()):
            bad |= 8
        bad |= _validate_vertices(n, root, lv, pa)
        return int(tmax(bad))

    for r in roots[: args.warmup]:
        dg.run(int(r), level, parent, **opts)
    clocks = ClockSampler(local)
    clocks.start()
    per, bad_roots = [], []
    alg = 0
    for r in roots[args.warmup:]:
        flush.fill_(1)
        torch.cuda.synchronize()
        comm.barrier()
        _, _, st = dg.run(int(r), level, parent, **opts)
        ms = tmax(st.elapsed_ms)                      # max over ranks of the device time
        if not args.no_validate:
            b = validate(int(r))
            if b:
                bad_roots.append((int(r), b))
        alg += metrics.d3_bytes(n, st.strategy, st.frontier_vertices, st.frontier_edges, st.unvisited, st.bu_probes)
        per.append((int(r), ms, st.input_edges_traversed, st.arcs_traversed, st.num_levels,
                    "".join("FSB"[s] for s in st.strategy), st.kernel_launches))
    clk = clocks.stop()
    if bad_roots:
        raise SystemExit(f"validation FAILED for timed roots {bad_roots[:5]}")
    # e2e: the same call, then each rank's level/parent slice into pinned host memory
    lh = torch.empty(max(dg.count, 1), dtype=torch.int32, pin_memory=True)[: dg.count]
    ph = torch.empty(max(dg.count, 1), dtype=torch.int32, pin_memory=True)[: dg.count]
    e2e = []
    m_of = {p[0]: p[2] for p in per}
    for r in roots[args.warmup: args.warmup + min(args.e2e_roots, args.steps)]:
        flush.fill_(1)
        torch.cuda.synchronize()
        comm.barrier()
        t1 = time.perf_counter()
        dg.run(int(r), level, parent, stats=False, **opts)
        lh.copy_(level)
        ph.copy_(parent)
        e2e.append(m_of[int(r)] / tmax(time.perf_counter() - t1))
    teps = [m / (ms * 1e-3) for (_, ms, m, *_r) in per]
    hm = metrics.harmonic_mean(teps)
    ms_mean = statistics.mean(p[1] for p in per)
    peak, peak_src = load_peaks()
    ach = alg / world / (sum(p[1] for p in per) * 1e-3) / 1e9
    if rank == 0:
        line = {
            "metric": METRIC, "value": round(hm / 1e9 / world, 3), "unit": "GTEPS", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_mean, 4), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic (seeded Graph500 Kronecker generator, graph seed 1, root seed 2; each rank "
                    "generates its own tuple share)",
            "config": bench_config(args, n, m_all, dg.arcs, world),
            "gteps_total": round(hm / 1e9, 3),
            "gteps_arcs_hmean": round(metrics.harmonic_mean([a / (ms * 1e-3) for (_, ms, _, a, *_r) in per]) / 1e9,
                                      3),
            "validated_roots": f"{len(per) - len(bad_roots)}/{len(per)}" if not args.no_validate else "skipped",
            "clocks": clk,
            "e2e": {"value": round(metrics.harmonic_mean(e2e) / 1e9 / world, 3) if e2e else None, "unit": "GTEPS",
                    "h2d_bytes_per_step": 8, "d2h_bytes_per_step": 8 * n,
                    "note": "xbfs_run_dist + every rank's level/parent slice D2H into pinned host memory, wall "
                            "clock (max over ranks), per B200"},
            "gpu_launches": int(sum(p[6] for p in per) * world),
            "roofline": {"bound": "hbm", "kernel": "xbfs_run_dist (whole BFS per rank)", "achieved": round(ach, 1),
                         "peak": peak, "unit": "GB/s", "frac": round(ach / peak, 4), "traffic": None,
                         "peak_source": peak_src,
                         "note": "SURVEY §8(d) D-3 bytes of the whole BFS / N per GPU / max-over-ranks device time "
                                 "(host collectives between levels included)"},
            "cpu_baseline": {"value": None, "kind": "oracle", "cores": None,
                             "sample": "rank 0 at N=1 only (bench contract); see the N=1 line"},
            "levels": [p[4] for p in per[:4]],
            "strategies": [rle(p[5]) for p in per[:4]],
            "prep_s": {"generate": round(t_gen, 2), "build_dist": round(t_build, 2)},
        }
        print(json.dumps(line), flush=True)
    dg.close()
    comm.close()
    dist.destroy_process_group()


# ---------------------------------------------------------------------------
# CPU oracle: cpu_baseline and the reference arm
# ---------------------------------------------------------------------------

def cpu_baseline(args, src, dst, n, roots, budget_s=None):
    """The oracle as it stands (serial FIFO BFS, 1 thread) on a bounded sample of
    the same workload: the first roots until ~budget seconds of BFS time."""
    import oracle
    from paper_conf_sc_yangls0w24_b200 import metrics
    budget_s = args.cpu_budget if budget_s is None else budget_s
    t0 = time.time()
    og = (oracle.build_csr_directed if CONFIGS[args.config].get("directed") else oracle.build_csr)(n, src, dst)
    t_csr = time.time() - t0
    teps, used, spent = [], [], 0.0
    for r in roots:
        t1 = time.perf_counter()
        lv, _, _ = oracle.bfs(og, int(r))
        dt = time.perf_counter() - t1
        teps.append(oracle.input_edges(src, lv) / dt)
        used.append(int(r))
        spent += dt
        if spent >= budget_s:
            break
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
    roots = pick_roots(args.config, n, src, dst, 4 * (args.warmup + args.steps) if directed
                       else args.warmup + args.steps)
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
        "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int32", "data": "synthetic",
        "config": bench_config(args, n, src.shape[0], og.arcs, world),
        "cpu_baseline": {"value": round(value, 5), "unit": "GTEPS", "cores": 1, "kind": "oracle",
                         "sample": f"{args.steps} roots, one full serial BFS each (oracle CSR prebuilt, untimed)"},
        "e2e": {"value": round(value, 5), "unit": "GTEPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------
# launcher
# ---------------------------------------------------------------------------

def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def launch(args) -> int:
    """`--gpus N` without torchrun: start N ranks of this script on 127.0.0.1."""
    if not args.launcher_selftest:
        import torch
        have = torch.cuda.device_count()
        if have < args.gpus:
            print(f"bench.py: --gpus {args.gpus} but only {have} CUDA device(s) visible", file=sys.stderr)
            return 1
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


def launcher_selftest(args):
    """Every rank joins a gloo group and the library communicator; rank 0 prints one line."""
    import torch.distributed as dist

    from paper_conf_sc_yangls0w24_b200.dist import Comm
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    c = Comm.from_torch()
    s = c.allreduce([rank + 1, 1]).tolist()
    ranks = [None] * world
    dist.all_gather_object(ranks, rank)
    if rank == 0:
        print(json.dumps({"n_ranks": world, "allreduce": s, "ranks": ranks}), flush=True)
    c.close()
    dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=64)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default=None, choices=sorted(CONFIGS),
                    help="default: s24 at N = 1, s27 (BASELINE config 4) at N > 1")
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
    ap.add_argument("--no-validate", action="store_true", help="skip the untimed per-root validation")
    ap.add_argument("--mode", default="auto", choices=["auto", "dist"],
                    help="dist at N = 1: the partitioned path on one GPU")
    ap.add_argument("--launcher-selftest", action="store_true", help=argparse.SUPPRESS)
    args = ap.parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(launch(args))
    if args.launcher_selftest:
        return launcher_selftest(args)
    if args.config is None:
        args.config = "s27" if world > 1 else "s24"
    assert args.warmup >= 3 or args.impl == "reference" or os.environ.get("XBFS_ALLOW_SHORT_WARMUP"), \
        "timing rules: at least 3 warm-up steps"
    if args.impl == "reference":
        run_reference(args)
    elif world > 1 or args.mode == "dist":
        run_dist(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()

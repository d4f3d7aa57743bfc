#!/usr/bin/env python
"""bench.py -- throughput of the batched point-by-tree traversal on B200.

Contract (driver):  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
N > 1 runs under torchrun (one process per GPU, NCCL).  Rank 0 prints ONE JSON line.

Workload (default, N=1): BASELINE.json configs[1] -- Barnes-Hut force pass over
a 1M-body Plummer sphere, theta = 0.5, eps = 0.05, fp32.  A step is one pass
of the hot path: tt_sort_points (key kernel + radix sort)
then tt_traverse_bh (per-warp mode choice, traversal, write-out in the
caller's order); for N > 1 also the all-gather of the results.  The tree
upload (a0) is timed separately (`upload_ms`), as §8(a) specifies.
Scaling is weak: every rank owns M = 1M bodies of an N*M-body Plummer sphere
whose tree is built on rank 0 and NCCL-broadcast.

metric = points traversed / s (whole job, all ranks); node visits / s and the
roofline of the dominant kernel are reported alongside.
--impl reference times the CPU oracle (the reference arm of this tier) on
the host cores, on a bounded sample of the same workload.
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

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import ttgen  # noqa: E402

METRIC = "points traversed/sec and node visits/sec at 1/2/4/8 B200; % HBM peak"
# SURVEY §8(d) algorithmic bytes per useful visit (kNN: 16 B per node visit
# plus 32 B per leaf-point distance, tt_stats.point_tests; NN, not in §8(d):
# its 16-B header + the node's 32-B point) and per point of I/O
BYTES_PER_VISIT = {"bh": 32, "pc": 32, "knn": 16, "vp": 80, "nn": 48}
BYTES_PER_POINT_TEST = {"knn": 32}
BYTES_PER_POINT_IO = {"bh": 32, "pc": 20, "knn": 28 + 64, "vp": 64 + 8, "nn": 28 + 8}
# bytes of one fetched node in our packed layout (record + the side rows read
# with it: kd boxes, kNN children's boxes, VP / NN points), for node_fetch
FETCH_BYTES = {"bh": 32, "pc": 32 + 32, "knn": 32 + 128, "vp": 16 + 64, "nn": 16 + 64 + 32}
L2_FLUSH_BYTES = 256 << 20  # 2x the 126 MB L2
# The paper's own numbers, other hardware (Tesla C2070: 14 SMs, vs 4 AMD
# Opteron 6176, 32 threads): context only, never a ratio.
PAPER_CONTEXT = {
    "bh": {"claim": "speedups of up to 38x over 32-thread CPU versions (P:L29-31)",
           "paper_traversal_ms": 669.07, "paper_visits_per_point": 3345,
           "paper_speedup_vs_32_threads": 7.18,
           "what": "Table 1, Barnes-Hut Plummer 1M bodies, sorted, lockstep (P:L1150)",
           "hardware": "NVIDIA Tesla C2070 vs 4x AMD Opteron 6176 (P:L1096-1108)"},
}


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--workload", choices=["bh", "knn", "vp", "pc", "nn", "bh16m", "knn16m", "bhsteps"], default="bh",
                    help="bh/knn/vp/pc: configs[0..3] (weak scaling, M points per rank); "
                         "bh16m/knn16m: configs[4] (16M points split over the ranks, strong scaling); "
                         "bhsteps: full BH time steps (GPU build + sort + force + leapfrog), bodies sharded over the ranks (strong scaling)")
    ap.add_argument("--mode", default="auto", choices=["auto", "lockstep", "independent"])
    ap.add_argument("--unsorted", action="store_true", help="skip tt_sort_points (paper's 'unsorted' column)")
    ap.add_argument("--no-schedule", action="store_true",
                    help="skip tt_schedule_tiles (longest-first tile order after the sort; kd/vp trees)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-chase", action="store_true", help="skip the live L2-latency (tt_diag_chase) roof")
    ap.add_argument("--points-per-rank", type=int, default=0, help="override M (testing)")
    ap.add_argument("--no-strong", action="store_true",
                    help="skip the fixed-config strong-scaling block (configs[4] BH 16M, every N)")
    ap.add_argument("--strong-points", type=int, default=0, help="override the strong block's N (testing)")
    ap.add_argument("--leaf", type=int, default=0, help="override the kd bucket size (tuning sweeps only)")
    ap.add_argument("--steps-order", default="sort", choices=["build", "sort"],
                    help="bhsteps traversal order: the GPU build's tree order, or tt_sort_points (Hilbert)")
    ap.add_argument("--auto-min-depth", type=int, default=None, help="AUTO-mode threshold (default: kernel's)")
    ap.add_argument("--switch-below", type=int, default=0,
                    help="kNN: dynamic L->N switch when fewer lanes are active (NEXT-3; 0 = never)")
    ap.add_argument("--device-build", action="store_true",
                    help="build the tree on the GPU (tt_build_oct_device / tt_build_kd_device) instead of host "
                         "build + upload")
    ap.add_argument("--variant", default="autoropes", choices=["autoropes", "recursive", "stack", "split", "groups", "ropes"],
                    help="recursive = the paper's naive recursive GPU baseline (ablation, N mode); "
                         "stack = explicit rope stacks, Fig.9b (ablation, BH and PC)")
    return ap.parse_args()


# ------------------------------------------------------------------ inputs
_T0 = time.time()


def _trace(msg: str):
    """Phase trace on stderr (TT_BENCH_TRACE=1), rank-prefixed."""
    if os.environ.get("TT_BENCH_TRACE"):
        print(f"[bench r{os.environ.get('RANK', '0')} +{time.time() - _T0:7.2f}s] {msg}", file=sys.stderr, flush=True)


def make_workload(name: str, world: int, per_rank: int = 0):
    """Global synthetic inputs (identical on every rank: seeded)."""
    if name == "bh16m":
        c = dict(ttgen.CONFIGS["bh_16m_plummer"])
        n = per_rank * world if per_rank else c["n"]
        data = ttgen.plummer(n, c["seed"])
        return dict(cfg=c, workload="bh_16m_plummer", data=data, queries=data, m=n // world, n_data=n,
                    strong=True)
    if name == "knn16m":
        c = dict(ttgen.CONFIGS["knn_16m_7d"])
        n = per_rank * world if per_rank else c["m"]
        data = ttgen.gaussian_mixture(c["n"], c["dim"], c["seed"])
        q = ttgen.gaussian_mixture(n, c["dim"], c["qseed"])
        return dict(cfg=c, workload="knn_16m_7d", data=data, queries=q, m=n // world, n_data=c["n"], strong=True)
    if name == "bh":
        c = dict(ttgen.CONFIGS["bh_1m_plummer"])
        m = per_rank or c["n"]
        data = ttgen.plummer(m * world, c["seed"])
        return dict(cfg=c, workload="bh_1m_plummer", data=data, queries=data, m=m, n_data=m * world)
    if name == "knn":
        c = dict(ttgen.CONFIGS["knn_1m_7d"])
        m = per_rank or c["m"]
        data = ttgen.gaussian_mixture(c["n"], c["dim"], c["seed"])
        q = ttgen.gaussian_mixture(m * world, c["dim"], c["qseed"])
        return dict(cfg=c, workload="knn_1m_7d", data=data, queries=q, m=m, n_data=c["n"])
    if name == "nn":  # NEXT-3: the paper's NN benchmark on configs[2]'s inputs
        c = dict(ttgen.CONFIGS["knn_1m_7d"])
        m = per_rank or c["m"]
        data = ttgen.gaussian_mixture(c["n"], c["dim"], c["seed"])
        q = ttgen.gaussian_mixture(m * world, c["dim"], c["qseed"])
        return dict(cfg=c, workload="nn_1m_7d (point-per-node kd-tree, configs[2] inputs)", data=data, queries=q,
                    m=m, n_data=c["n"])
    if name == "vp":
        c = dict(ttgen.CONFIGS["vp_1m_16d"])
        m = per_rank or c["m"]
        data = ttgen.gaussian_mixture(c["n"], c["dim"], c["seed"])
        q = ttgen.gaussian_mixture(m * world, c["dim"], c["qseed"])
        return dict(cfg=c, workload="vp_1m_16d", data=data, queries=q, m=m, n_data=c["n"])
    c = dict(ttgen.CONFIGS["pc_10k_3d"])
    m = per_rank or c["n"]
    data = ttgen.uniform(c["n"], c["dim"], c["seed"])
    q = data if world == 1 and m == c["n"] else ttgen.uniform(m * world, c["dim"], c["seed"] + 100)
    return dict(cfg=c, workload="pc_10k_3d", data=data, queries=q, m=m, n_data=c["n"])


def host_tree(P, name, w):
    c = w["cfg"]
    if name == "bh":
        return P.build_oct(w["data"])
    if name == "vp":
        return P.build_vp(w["data"])
    if name == "nn":
        return P.build_nn(w["data"])
    return P.build_kd(w["data"], c["leaf"])


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md)."""
    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits", "-lms", "100",
                 "-i", str(self.gpu)], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            # nvidia-smi's start-up (NVML init) takes driver locks that stall
            # this process's CUDA API calls: let it reach its first sample
            # before the caller starts the timed region
            t0 = time.time()
            while not self.lines and self.proc.poll() is None and time.time() - t0 < 10:
                time.sleep(0.01)
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 9:
                continue
            try:
                sm.append(float(f[1]))
                mx.append(float(f[2]))
            except ValueError:
                continue
            for nm, v in zip(names, f[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        if not sm:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"], "samples": 0}
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": max(mx), "reasons": sorted(reasons),
                "samples": len(sm)}


# ------------------------------------------------------------ kernel count
def count_kernels(step_fn) -> int | None:
    """Kernels launched by one step, counted from a CUDA-graph capture of it."""
    import torch
    try:
        from cuda.bindings import runtime as rt
        g = torch.cuda.CUDAGraph(keep_graph=True)
        s = torch.cuda.Stream()
        torch.cuda.synchronize()
        with torch.cuda.stream(s):
            g.capture_begin()
            step_fn()
            g.capture_end()
        torch.cuda.synchronize()
        raw = g.raw_cuda_graph()
        err, _, n = rt.cudaGraphGetNodes(rt.cudaGraph_t(init_value=raw), 0)
        err, nodes, n = rt.cudaGraphGetNodes(rt.cudaGraph_t(init_value=raw), n)
        k = 0
        for nd in nodes:
            e, ty = rt.cudaGraphNodeGetType(nd)
            if ty == rt.cudaGraphNodeType.cudaGraphNodeTypeKernel:
                k += 1
        del g
        return k
    except Exception as e:  # capture not possible: reported as null
        print(f"[bench] kernel count via graph capture failed: {e!r}", file=sys.stderr)
        torch.cuda.synchronize()
        return None


def load_counts(workload: str, mode: str):
    """Per-point DRAM bytes and executed warp instructions of the traversal
    kernel from the committed `ncu --set full` capture (profiles/ncu_counts.json,
    written by tools/make_profiles.py), if any."""
    path = os.path.join(ROOT, "profiles", "ncu_counts.json")
    try:
        return json.load(open(path)).get(f"{workload}/{mode}")
    except (OSError, ValueError):
        return None


KERNEL_SOURCE = {"bh": ["kern_bh_group.cu"], "pc": ["kern_pc.cu", "kern_pc_split.cu"], "knn": ["kern_knn.cu"],
                 "vp": ["kern_vp.cu"], "nn": ["kern_nn.cu"]}


def kernel_sha256(workload: str) -> str:
    """Hash of the sources that decide the traversal kernel's instruction
    stream for `workload` (its kern_*.cu, the shared device headers and the
    nvcc flags of build.py); nvcc output bytes themselves are not
    reproducible."""
    import hashlib
    kind = workload.rstrip("0123456789m").replace("steps", "")  # bh16m -> bh, bhsteps -> bh
    pkg = os.path.join(ROOT, "paper_conf_sc_goldfarbjk13_b200")
    files = [os.path.join(pkg, "csrc", f) for f in (*KERNEL_SOURCE[kind], "kern_common.cuh", "tt_internal.h")]
    h = hashlib.sha256()
    for f in files:
        h.update(os.path.basename(f).encode())
        h.update(open(f, "rb").read())
    # the compile flags of build.py (not its source list)
    flags = [ln.strip() for ln in open(os.path.join(pkg, "build.py")).read().splitlines()
             if "ARCH" in ln or "-O3" in ln or "-Xptxas" in ln or "-lineinfo" in ln]
    h.update("\n".join(flags).encode())
    return h.hexdigest()


def chase_ceiling(P, nrec: int, device, per_lane: bool, steps: int = 3000) -> float:
    """Dependent record loads per second of a pure chase (tt_diag_chase):
    the walk's latency ceiling.  Median of 3 timed launches after 1 warm-up."""
    import torch
    rec = P.chase_records(int(nrec), device)
    nsm = torch.cuda.get_device_properties(device).multi_processor_count
    chains = nsm * 4 * 256 if per_lane else nsm * 4 * 8
    n = steps // 8 if per_lane else steps
    s = torch.cuda.current_stream()
    P.tt_diag_chase(rec, n, per_lane)
    ts = []
    for _ in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        P.tt_diag_chase(rec, n, per_lane)
        b.record(s)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) / 1e3)
    del rec
    return chains * n / statistics.median(ts)


def l2_ceiling(P, device, nbytes: int = 64 << 20, reps: int = 20) -> float:
    """L2 read GB/s of an L2-resident buffer (tt_diag_l2read), median of 3."""
    import torch
    buf = torch.ones(nbytes // 4, dtype=torch.float32, device=device)
    s = torch.cuda.current_stream()
    P.tt_diag_l2read(buf, reps)
    ts = []
    for _ in range(3):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        P.tt_diag_l2read(buf, reps)
        b.record(s)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) / 1e3)
    del buf
    return nbytes * reps / statistics.median(ts) / 1e9


def measured_peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json"))), "measured"
    except (OSError, ValueError):
        return {"hbm_gbs": 6650.0}, "fallback"


# ----------------------------------------------------------- oracle timing
def oracle_baseline(name, w, budget_points=None):
    """The oracle as it stands, on the host cores, on a bounded sample."""
    import oracle
    c = w["cfg"]
    q = w["queries"]
    m = len(q)
    # sample sized for ~10-30 s of CPU work: every frac-th query
    target = {"bh": 500_000, "knn": 125_000, "vp": 2_000, "pc": 10_000, "nn": 125_000}[name]
    frac = max(1, m // target)
    idx = np.arange(0, m, frac)
    if budget_points:
        idx = idx[:budget_points]
    threads = oracle.max_threads()
    if name == "bh":
        t = oracle.build_oct(w["data"])
        t0 = time.perf_counter()
        oracle.bh(t, q[idx], c["theta"], c["eps"], self_ids=idx, threads=threads)
    elif name == "knn":
        t = oracle.build_kd(w["data"], c["leaf"])
        t0 = time.perf_counter()
        oracle.knn(t, q[idx], c["k"], threads=threads)
    elif name == "vp":
        t = oracle.build_vp(w["data"])
        t0 = time.perf_counter()
        oracle.vp(t, q[idx], threads=threads)
    elif name == "nn":
        t = oracle.build_nn(w["data"])
        t0 = time.perf_counter()
        oracle.nn(t, q[idx], threads=threads)
    else:
        t = oracle.build_kd(w["data"], c["leaf"])
        t0 = time.perf_counter()
        oracle.pc(t, q[idx], c["radius"], threads=threads)
    dt = time.perf_counter() - t0
    return {"value": len(idx) / dt, "unit": "points/s", "cores": threads, "kind": "oracle",
            "sample": f"every {frac}th query ({len(idx)} of {m}) over the full tree; tree build excluded",
            "seconds": dt}


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle on this box's host cores (rank 0 only)."""
    if rank != 0:
        return
    w = make_workload(args.workload, 1, args.points_per_rank)
    name = {"bh16m": "bh", "knn16m": "knn"}.get(args.workload, args.workload)
    vals = []
    for _ in range(max(1, min(args.steps, 3))):
        vals.append(oracle_baseline(name, w))
    v = statistics.median(x["value"] for x in vals)
    cb = dict(vals[0])
    cb["value"] = v
    line = {"impl": "reference", "metric": METRIC, "value": v, "unit": "points/s", "n_gpus": world,
            "steps": len(vals), "warmup": 0, "ms_per_step": 1000.0 * statistics.median(x["seconds"] for x in vals),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32 decisions / f64 BH sums",
            "data": "synthetic", "config": {"workload": w["workload"], "points": len(w["queries"])},
            "cpu_baseline": cb, "e2e": {"value": v, "unit": "points/s", "h2d_bytes_per_step": 0,
                                         "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------- ours
def run_bh_steps(args, rank, world):
    """NEXT-4 workload: a bench step = one BH time step of configs[1]
    (tt_build_oct_device_order + tt_sort_points + tt_traverse_bh + tt_kick_drift_permuted,
    + all-gather of positions / velocities / ids for N > 1).  Strong scaling:
    the same 1M-body system on every N; each rank integrates its warp-aligned
    shard of the sorted order (nbody.simulate_sharded)."""
    import torch
    import torch.distributed as dist
    from paper_conf_sc_goldfarbjk13_b200 import nbody
    from paper_conf_sc_goldfarbjk13_b200 import parallel as PAR
    c = dict(ttgen.CONFIGS["bh_1m_plummer"])
    n = args.points_per_rank or c["n"]
    n = -(-n // (64 * world)) * (64 * world)  # equal warp-aligned shards
    b = ttgen.plummer(n, c["seed"])
    v = ttgen.plummer_velocities(b, c["seed"] + 1000)
    dev = torch.device("cuda", torch.cuda.current_device())
    B, V = torch.from_numpy(b).to(dev), torch.from_numpy(v).to(dev)
    ids = torch.arange(n, dtype=torch.int32, device=dev)
    dt = 1e-3
    for _ in range(args.warmup):
        B, V, ids = nbody.simulate_sharded(B, V, ids, 1, dt, c["theta"], c["eps"], final_kick=False,
                                           order=args.steps_order)
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    with ClockSampler(torch.cuda.current_device()) as clk:
        for i in range(args.steps):
            evs[i][0].record(stream)
            B, V, ids = nbody.simulate_sharded(B, V, ids, 1, dt, c["theta"], c["eps"], final_kick=False,
                                               order=args.steps_order)
            evs[i][1].record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    ms = statistics.mean(a.elapsed_time(b_) for a, b_ in evs)
    if world > 1:
        ms = PAR.max_over_ranks(ms, dev)
    if rank != 0:
        return
    line = {"metric": METRIC, "value": n / (ms / 1e3), "unit": "points/s (body-steps/s)", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": "bh_1m_plummer time steps", "bodies": n, "dt": dt, "order": args.steps_order,
                       "step": "GPU build + sort + force (own shard) + gathered kick-drift (leapfrog KDK)"
                               + (" + all-gather of x, v, ids" if world > 1 else ""),
                       "parallelism": f"dp{world} (bodies sharded by sorted order, tree rebuilt on every rank)",
                       "params": c, "l2": "not flushed: a time step rewrites the bodies and rebuilds the tree"},
            "clocks": clk.summary()}
    print(json.dumps(line), flush=True)


def run_strong16m(args, rank, world, device, P, PAR, kind="bh"):
    """configs[4]: one fixed problem at every N -- strong scaling.  kind "bh":
    the 16M-body Plummer sphere, theta 0.5; kind "knn": k = 8 for 16M 7-D
    queries over 16M 7-D mixture points.  Rank 0 builds the tree on its GPU
    (tt_build_{oct,kd}_device, NEXT-1) and NCCL-broadcasts the packed blob
    (tt_tree_copy_blob -> broadcast -> tt_tree_from_blob); every rank places
    the points in global sorted order once (data placement) and owns a
    contiguous warp-aligned range; a timed step = a1 sort of the rank's shard
    (+ a1b tile schedule for kNN) + traversal + all-gather of the results.
    Each phase is reported separately; every time is the max over ranks
    (CUDA events)."""
    import torch
    import torch.distributed as dist
    c = ttgen.CONFIGS["bh_16m_plummer" if kind == "bh" else "knn_16m_7d"]
    n = args.strong_points or (c["n"] if kind == "bh" else c["m"])
    if world > 1 and n % (64 * world):
        raise SystemExit(f"bench: {n} points do not split into {world} equal warp-aligned shards")
    ids_shard = None
    if kind == "bh":
        data = ttgen.plummer(n, c["seed"])
        queries = data
    else:
        data = ttgen.gaussian_mixture(args.strong_points or c["n"], c["dim"], c["seed"])
        queries = ttgen.gaussian_mixture(n, c["dim"], c["qseed"])
    d_all = torch.from_numpy(np.ascontiguousarray(data)).to(device)
    _trace(f"strong {kind}: inputs ready")
    stream = torch.cuda.current_stream()
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    tree = None
    if rank == 0:
        tree = P.tt_build_oct_device(d_all) if kind == "bh" else P.tt_build_kd_device(d_all, c["leaf"])
    torch.cuda.synchronize()
    build_ms = 1e3 * (time.perf_counter() - t0)
    _trace(f"strong {kind}: built")
    bcast_ms = None
    if world > 1:
        dist.barrier()
        t0 = time.perf_counter()
        tree = PAR.broadcast_device_tree(tree, device)
        torch.cuda.synchronize()
        bcast_ms = PAR.max_over_ranks(1e3 * (time.perf_counter() - t0), device)
    q_all = d_all if kind == "bh" else torch.from_numpy(np.ascontiguousarray(queries)).to(device)
    del d_all
    t0 = time.perf_counter()
    gperm = P.tt_sort_points(tree, q_all).long()
    q = q_all[gperm].contiguous()
    ids = gperm.to(torch.int32)
    del q_all, gperm
    torch.cuda.synchronize()
    placement_ms = 1e3 * (time.perf_counter() - t0)
    _trace(f"strong {kind}: placed")
    if kind == "bh":
        outs = (torch.zeros((n, 4), dtype=torch.float32, device=device),)
    else:
        outs = (torch.zeros((n, c["k"]), dtype=torch.int32, device=device),
                torch.zeros((n, c["k"]), dtype=torch.float32, device=device))

    def run(qs, oslices, order, stats=None):
        if kind == "bh":
            P.tt_traverse_bh(tree, qs, c["theta"], c["eps"], out=oslices[0], self_ids=ids_shard, order=order,
                             stats=stats)
        else:
            P.tt_traverse_knn(tree, qs, c["k"], out_idx=oslices[0], out_d2=oslices[1], order=order, stats=stats)

    # Cost-balanced shards: every rank traverses its
    # equal-count shard once with stats (untimed), the per-point visit counts
    # are all-gathered, and the shard boundaries are put where their prefix
    # sum crosses r/N of the total (warp-aligned); results then travel by a
    # padded all-gather.  N = 1: one shard.
    ranges = [(0, n)]
    imb_equal = imb_bal = 1.0
    if world > 1:
        lo, hi = PAR.shard_range(n, rank, world)
        ids_shard = ids[lo:hi]
        order = P.tt_sort_points(tree, q[lo:hi])
        st = P.Stats.alloc(hi - lo, device)
        run(q[lo:hi], tuple(o[lo:hi] for o in outs), order, st)
        vis = torch.zeros((n, 1), dtype=torch.int32, device=device)
        vis[lo:hi, 0] = st.visits
        PAR.allgather_rows(vis, world)
        cost = vis[:, 0].to(torch.float64)
        ranges = PAR.balanced_ranges(cost, world)
        per = lambda rs: [float(cost[a:b].sum()) for a, b in rs]  # noqa: E731
        eq = per([PAR.shard_range(n, r, world) for r in range(world)])
        bal = per(ranges)
        imb_equal, imb_bal = max(eq) / (sum(eq) / world), max(bal) / (sum(bal) / world)
        del st, vis, cost
    lo, hi = ranges[rank]
    q_shard, ids_shard = q[lo:hi], ids[lo:hi]
    order = torch.empty(hi - lo, dtype=torch.int32, device=device)
    lpt = kind == "knn" and (hi - lo) // 32 > 148 * 32

    def step(ev=None):
        if ev:
            ev[0].record(stream)
        P.tt_sort_points(tree, q_shard, out=order)
        if lpt:
            P.tt_schedule_tiles(tree, q_shard, order, out=order)
        if ev:
            ev[1].record(stream)
        run(q_shard, tuple(o[lo:hi] for o in outs), order)
        if ev:
            ev[2].record(stream)
        if world > 1:
            for o in outs:
                PAR.allgather_rows_var(o, ranges)
        if ev:
            ev[3].record(stream)

    for _ in range(args.warmup):
        step()
    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=device)
    evs = [[torch.cuda.Event(enable_timing=True) for _ in range(4)] for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for i in range(args.steps):
        flush.zero_()
        step(evs[i])
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    _trace(f"strong {kind}: timed")
    mean = lambda a, b: statistics.mean(e[a].elapsed_time(e[b]) for e in evs)  # noqa: E731
    ms, sort_ms, trav_ms, ag_ms = mean(0, 3), mean(0, 1), mean(1, 2), mean(2, 3)
    if world > 1:
        ms, sort_ms, trav_ms, ag_ms, placement_ms = (PAR.max_over_ranks(x, device) for x in
                                                     (ms, sort_ms, trav_ms, ag_ms, placement_ms))
    del flush, outs, q, ids
    return {"workload": "bh_16m_plummer" if kind == "bh" else "knn_16m_7d", "scaling": "strong",
            "value": n / (ms / 1e3), "unit": "points/s",
            "ms_per_step": ms, "sort_ms": sort_ms, "traverse_ms": trav_ms,
            "allgather_ms": ag_ms if world > 1 else None, "points": n, "points_per_rank": hi - lo,
            "tree_build_ms": build_ms,
            "tree_build": f"device (tt_build_{'oct' if kind == 'bh' else 'kd'}_device) on rank 0",
            "bcast_ms": bcast_ms, "placement_ms": placement_ms,
            "shards": "cost-balanced: prefix sum of a previous pass's per-point visit counts, warp-aligned"
                      if world > 1 else "one",
            "shard_cost_max_over_mean": {"equal_count": round(imb_equal, 4), "balanced": round(imb_bal, 4)},
            "note": "configs[4] at every N: step = a1 sort of the rank's shard (+ LPT schedule, kNN) + traversal "
                    "+ all-gather; build, broadcast and placement outside the timed steps, reported here"}


def run_ours(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist
    import paper_conf_sc_goldfarbjk13_b200 as P
    from paper_conf_sc_goldfarbjk13_b200 import parallel as PAR

    gpu = local_rank % torch.cuda.device_count()  # test mode may put ranks on one GPU
    torch.cuda.set_device(gpu)
    device = torch.device("cuda", gpu)
    w = make_workload(args.workload, world, args.points_per_rank)
    name = {"bh16m": "bh", "knn16m": "knn"}.get(args.workload, args.workload)
    c = w["cfg"]
    if args.leaf:
        c["leaf"] = args.leaf
    m = w["m"]
    if world > 1 and len(w["queries"]) % (64 * world):
        raise SystemExit(f"bench: {len(w['queries'])} points do not split into {world} equal warp-aligned "
                         "shards (the in-place all-gather needs n % (64 * N) == 0)")
    lo, hi = PAR.shard_range(len(w["queries"]), rank, world)
    m = hi - lo  # warp-aligned equal shards

    _trace("workload ready")
    # a0: tree (rank 0 builds; NCCL broadcast for N > 1) -- timed separately
    t0 = time.perf_counter()
    if args.device_build:
        # every rank builds the identical tree from the identical points (NEXT-1)
        data_dev = torch.from_numpy(np.ascontiguousarray(w["data"])).to(device)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        tree = (P.tt_build_oct_device(data_dev) if name == "bh"
                else P.tt_build_vp_device(data_dev) if name == "vp"
                else P.tt_build_nn_device(data_dev) if name == "nn"
                else P.tt_build_kd_device(data_dev, w["cfg"]["leaf"]))
        t1 = time.perf_counter()
        del data_dev
    elif world == 1:
        host = host_tree(P, name, w)
        t1 = time.perf_counter()
        tree = P.tt_tree_upload(host)
    else:
        host = host_tree(P, name, w) if rank == 0 else None
        t1 = time.perf_counter()
        tree = PAR.broadcast_tree(host, device)
    torch.cuda.synchronize()
    t2 = time.perf_counter()
    build_ms, upload_ms = 1e3 * (t1 - t0), 1e3 * (t2 - t1)
    _trace("tree ready")
    # a0 also includes BH's child-group array, derived from the uploaded blob
    # by the first traversal (kern_bh_group.cu): triggered and timed here, so
    # it is neither hidden in a traversal time nor left out of a0
    group_build_ms = None
    if name == "bh" and args.variant in ("autoropes", "groups"):
        qq = torch.from_numpy(np.ascontiguousarray(w["queries"][:64])).to(device)
        # the first launch of each kernel in a process pays its lazy module
        # load (hundreds of ms): warm them on a throwaway 64-body tree so the
        # time below is the group build itself
        tiny = P.tt_tree_upload(P.build_oct(np.ascontiguousarray(w["queries"][:64])))
        P.tt_traverse_bh(tiny, qq, c["theta"], c["eps"], mode="lockstep")
        torch.cuda.synchronize()
        del tiny
        t3 = time.perf_counter()
        P.tt_traverse_bh(tree, qq, c["theta"], c["eps"], mode="lockstep")
        torch.cuda.synchronize()
        group_build_ms = 1e3 * (time.perf_counter() - t3)
        del qq
    build_where = "device (tt_build_*_device)" if args.device_build else "host (tt_build_*)"

    q_all = torch.from_numpy(np.ascontiguousarray(w["queries"])).to(device)
    ids_all = None
    bcast_ms = upload_ms if world > 1 and not args.device_build else None
    torch.cuda.synchronize()
    t_pl = time.perf_counter()
    if world > 1 and not args.unsorted:
        # Spatial decomposition (data placement, before the timed region, as a
        # time-stepping code keeps its bodies -- DESIGN.md §9): rank r owns a
        # contiguous range of the global tree order, so its warps are as
        # coherent as on one GPU.  Each step still sorts the rank's own shard.
        gperm = P.tt_sort_points(tree, q_all).long()
        q_all = q_all[gperm].contiguous()
        ids_all = gperm.to(torch.int32)
    q_shard = q_all[lo:hi]
    torch.cuda.synchronize()
    placement_ms = 1e3 * (time.perf_counter() - t_pl) if world > 1 and not args.unsorted else None
    n_all = len(w["queries"])
    stream = torch.cuda.current_stream()
    order_buf = torch.empty(m, dtype=torch.int32, device=device)
    if name == "bh":
        out = torch.zeros((n_all, 4), dtype=torch.float32, device=device)
    elif name == "knn":
        out = (torch.zeros((n_all, c["k"]), dtype=torch.int32, device=device),
               torch.zeros((n_all, c["k"]), dtype=torch.float32, device=device))
    elif name in ("vp", "nn"):
        out = (torch.zeros(n_all, dtype=torch.int32, device=device),
               torch.zeros(n_all, dtype=torch.float32, device=device))
    else:
        out = torch.zeros(n_all, dtype=torch.int32, device=device)

    # shard views: the rank's points and result rows [lo, hi); BH self ids are
    # the bodies' global indices (the tree is built over all N*M bodies)
    def views(o):
        return tuple(x[lo:hi] for x in o) if isinstance(o, tuple) else o[lo:hi]

    out_shard = views(out)
    self_ids = None
    if name == "bh":  # the bodies' ids in the tree (original indices)
        self_ids = ids_all[lo:hi] if ids_all is not None else torch.arange(lo, hi, dtype=torch.int32, device=device)

    def traverse(pts, res, order, stats=None, mode=None):
        mode = mode or args.mode
        if name == "bh":
            P.tt_traverse_bh(tree, pts, c["theta"], c["eps"], out=res, self_ids=self_ids, order=order,
                             mode=mode, auto_min_depth=args.auto_min_depth, stats=stats,
                             variant=args.variant)
        elif name == "knn":
            P.tt_traverse_knn(tree, pts, c["k"], out_idx=res[0], out_d2=res[1], order=order, mode=mode,
                              auto_min_depth=args.auto_min_depth, stats=stats, variant=args.variant,
                              switch_below=args.switch_below)
        elif name == "vp":
            P.tt_traverse_vp(tree, pts, out_idx=res[0], out_d2=res[1], order=order, mode=mode,
                             auto_min_depth=args.auto_min_depth, stats=stats, variant=args.variant)
        elif name == "nn":
            P.tt_traverse_nn(tree, pts, out_idx=res[0], out_d2=res[1], order=order, mode=mode,
                             auto_min_depth=args.auto_min_depth, stats=stats)
        else:
            P.tt_traverse_pc(tree, pts, c["radius"], out=res, order=order, mode=mode,
                             auto_min_depth=args.auto_min_depth, stats=stats, variant=args.variant)

    if args.unsorted:
        order_buf.copy_(torch.arange(m, dtype=torch.int32, device=device))

    # a1b pays only when there are more tiles than resident warps (148 SMs x 32)
    lpt = not args.unsorted and not args.no_schedule and tree.kind != "oct" and m // 32 > 148 * 32

    def step(kev=None, collective=True, agev=None):
        if not args.unsorted:
            P.tt_sort_points(tree, q_shard, out=order_buf)  # a1
            if lpt:
                P.tt_schedule_tiles(tree, q_shard, order_buf, out=order_buf)  # a1b
        if kev:
            kev[0].record(stream)
        traverse(q_shard, out_shard, order_buf)            # a2-a5
        if kev:
            kev[1].record(stream)
        if world > 1 and collective:
            if agev:
                agev[0].record(stream)
            for o in (out if isinstance(out, tuple) else (out,)):
                PAR.allgather_rows(o, world)
            if agev:
                agev[1].record(stream)

    clk = ClockSampler(gpu).__enter__()
    # stats pass (untimed): per-point useful visits, warp fetches, modes
    if not args.unsorted:
        P.tt_sort_points(tree, q_shard, out=order_buf)
        if lpt:
            P.tt_schedule_tiles(tree, q_shard, order_buf, out=order_buf)
    st = P.Stats.alloc(m, device, point_tests=name in BYTES_PER_POINT_TEST)
    traverse(q_shard, out_shard, order_buf, st)
    torch.cuda.synchronize()
    visits = int(st.visits.to(torch.int64).sum().item())
    ptests = int(st.point_tests.to(torch.int64).sum().item()) if st.point_tests is not None else 0
    tile_pts = P._lib.TILE_POINTS[tree.kind] if args.variant in ("autoropes", "groups", "ropes") else 32
    tiles = -(-m // tile_pts)
    wf = int(st.warp_fetches[:tiles].to(torch.int64).sum().item())
    lock_frac = float((st.warp_mode[:tiles] == 1).float().mean().item())
    # Table 2's work expansion (reading R22): per lockstep warp
    # tile, the nodes the warp tested / the longest independent traversal of
    # its points (an extra, untimed independent-mode stats pass)
    we_table2 = None
    if lock_frac > 0 and args.variant in ("autoropes", "groups", "ropes"):
        sn = P.Stats.alloc(m, device)
        traverse(q_shard, out_shard, order_buf, sn, mode="independent")
        torch.cuda.synchronize()
        lanes = order_buf.long() if not args.unsorted else torch.arange(m, device=device)
        vn = sn.visits.to(torch.float64)[lanes]
        vn = torch.cat([vn, torch.zeros(tiles * tile_pts - m, dtype=torch.float64, device=device)])
        longest = vn.view(tiles, tile_pts).max(1).values
        lk = st.warp_mode[:tiles] == 1
        tested = st.warp_steps[:tiles].to(torch.float64)
        we_table2 = float((tested[lk] / longest[lk].clamp(min=1)).mean().item())
        del sn, vn
    del st

    _trace("stats pass done")
    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()
    _trace("warm-up done")
    # our kernels per step (the NCCL all-gather of N > 1 is not ours: excluded)
    launches = count_kernels(lambda: step(collective=False)) if rank == 0 else None

    flush = torch.empty(L2_FLUSH_BYTES // 4, dtype=torch.float32, device=device)
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    kevs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    agevs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for i in range(args.steps):
        flush.zero_()  # L2 flush between timed iterations (outside the events)
        evs[i][0].record(stream)
        step(kevs[i], agev=agevs[i])
        evs[i][1].record(stream)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in evs]
    kern_ms = [a.elapsed_time(b) for a, b in kevs]
    ms = statistics.mean(step_ms)
    kms = statistics.mean(kern_ms)
    allgather_ms = statistics.mean(a.elapsed_time(b) for a, b in agevs) if world > 1 else None
    if world > 1:
        ms = PAR.max_over_ranks(ms, device)
        kms = PAR.max_over_ranks(kms, device)
        allgather_ms = PAR.max_over_ranks(allgather_ms, device)
        if bcast_ms is not None:
            bcast_ms = PAR.max_over_ranks(bcast_ms, device)
        if placement_ms is not None:
            placement_ms = PAR.max_over_ranks(placement_ms, device)
        visits_all = torch.tensor([visits], dtype=torch.int64, device=PAR._wire(device))
        dist.all_reduce(visits_all)
        visits_tot = int(visits_all.item())
    else:
        visits_tot = visits

    # e2e through the public API with host buffers (pinned), copies inside
    e2e = None
    if not args.no_e2e:
        q_host = q_shard.cpu().pin_memory()
        q_dev = torch.empty_like(q_host, device=device)
        res_host = None
        if name == "bh":
            res_dev = torch.empty((m, 4), dtype=torch.float32, device=device)
            res_host = torch.empty((m, 4), dtype=torch.float32).pin_memory()
        elif name in ("knn",):
            res_dev = (torch.empty((m, c["k"]), dtype=torch.int32, device=device),
                       torch.empty((m, c["k"]), dtype=torch.float32, device=device))
            res_host = tuple(torch.empty(r.shape, dtype=r.dtype).pin_memory() for r in res_dev)
        elif name in ("vp", "nn"):
            res_dev = (torch.empty(m, dtype=torch.int32, device=device),
                       torch.empty(m, dtype=torch.float32, device=device))
            res_host = tuple(torch.empty(r.shape, dtype=r.dtype).pin_memory() for r in res_dev)
        else:
            res_dev = torch.empty(m, dtype=torch.int32, device=device)
            res_host = torch.empty(m, dtype=torch.int32).pin_memory()
        perm = torch.empty(m, dtype=torch.int32, device=device)

        def api_step(qd, rd, pm):
            """One step through the public API on the current stream."""
            P.tt_sort_points(tree, qd, out=pm)
            if lpt:
                P.tt_schedule_tiles(tree, qd, pm, out=pm)
            if name == "bh":
                P.tt_traverse_bh(tree, qd, c["theta"], c["eps"], out=rd, order=pm, mode=args.mode,
                                 self_ids=self_ids)
            elif name == "knn":
                P.tt_traverse_knn(tree, qd, c["k"], out_idx=rd[0], out_d2=rd[1], order=pm, mode=args.mode)
            elif name in ("vp", "nn"):
                (P.tt_traverse_vp if name == "vp" else P.tt_traverse_nn)(
                    tree, qd, out_idx=rd[0], out_d2=rd[1], order=pm, mode=args.mode)
            else:
                P.tt_traverse_pc(tree, qd, c["radius"], out=rd, order=pm, mode=args.mode)

        def to_host(rh, rd):
            for h_, d_ in zip(rh if isinstance(rh, tuple) else (rh,), rd if isinstance(rd, tuple) else (rd,)):
                h_.copy_(d_, non_blocking=True)

        def e2e_step():  # serialised: H2D, sort, traversal, D2H on one stream
            q_dev.copy_(q_host, non_blocking=True)
            api_step(q_dev, res_dev, perm)
            to_host(res_host, res_dev)

        for _ in range(2):
            e2e_step()
        torch.cuda.synchronize()
        ee = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        for i in range(args.steps):
            flush.zero_()
            ee[i][0].record(stream)
            e2e_step()
            ee[i][1].record(stream)
        torch.cuda.synchronize()
        serial_ms = statistics.mean(a.elapsed_time(b) for a, b in ee)

        # Streamed: the copies of step i overlap the traversal of step i-1 /
        # i+1 (a copy stream, two device buffer sets); every step still copies
        # its inputs in and its results out, and each step's compute is
        # preceded (inside the timed region) by the L2 flush.
        like = lambda r: tuple(torch.empty_like(x) for x in r) if isinstance(r, tuple) else torch.empty_like(r)  # noqa: E731
        qds, rds, pms = [q_dev, torch.empty_like(q_dev)], [res_dev, like(res_dev)], [perm, torch.empty_like(perm)]
        rhs = [res_host, tuple(torch.empty(x.shape, dtype=x.dtype).pin_memory() for x in res_host)
               if isinstance(res_host, tuple) else torch.empty(res_host.shape, dtype=res_host.dtype).pin_memory()]
        # separate H2D and D2H streams: the next step's H2D must not queue
        # behind this step's D2H (which waits for this step's compute)
        cs, ds = torch.cuda.Stream(device), torch.cuda.Stream(device)
        ev = lambda: torch.cuda.Event()  # noqa: E731
        h2d_done, comp_done, d2h_done = [ev(), ev()], [ev(), ev()], [ev(), ev()]

        def pipe_step(i):
            b_ = i % 2
            with torch.cuda.stream(cs):
                cs.wait_event(comp_done[b_])          # step i-2 done reading qds[b_]
                qds[b_].copy_(q_host, non_blocking=True)
                h2d_done[b_].record(cs)
            stream.wait_event(h2d_done[b_])
            stream.wait_event(d2h_done[b_])           # step i-2's results copied out of rds[b_]
            flush.zero_()
            api_step(qds[b_], rds[b_], pms[b_])
            comp_done[b_].record(stream)
            with torch.cuda.stream(ds):
                ds.wait_event(comp_done[b_])
                to_host(rhs[b_], rds[b_])
                d2h_done[b_].record(ds)

        for i in range(4):
            pipe_step(i)
        torch.cuda.synchronize()
        t_a, t_b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        t_a.record(stream)
        cs.wait_stream(stream)
        ds.wait_stream(stream)
        for i in range(args.steps):
            pipe_step(i)
        for b_ in range(2):
            stream.wait_event(d2h_done[b_])
        t_b.record(stream)
        torch.cuda.synchronize()
        ems = t_a.elapsed_time(t_b) / args.steps
        if world > 1:
            ems = PAR.max_over_ranks(ems, device)
            serial_ms = PAR.max_over_ranks(serial_ms, device)
        d2h = sum(r.numel() * r.element_size() for r in (res_host if isinstance(res_host, tuple) else (res_host,)))
        e2e = {"value": n_all / (ems / 1e3), "unit": "points/s", "ms_per_step": ems,
               "h2d_bytes_per_step": int(q_host.numel() * q_host.element_size()), "d2h_bytes_per_step": int(d2h),
               "serial_ms_per_step": serial_ms,
               "note": "public API (tt_sort_points + tt_schedule_tiles + tt_traverse_*) from / to pinned host "
                       "buffers: every step copies its points in (H2D) and its results out (D2H); the copies run "
                       "on two copy streams, overlapping the neighbouring steps' compute (double-buffered); "
                       "L2 flushed before each step's compute inside the timed region.  serial_ms_per_step: "
                       "the same with H2D, compute and D2H serialised on one stream"}

    # keep the GPU busy until the sampler has seen the load (>= 5 samples)
    t_soak = time.perf_counter()
    while len(clk.lines) < 5 and time.perf_counter() - t_soak < 3.0:
        step(collective=False)  # rank-local: the ranks may soak a different number of steps
        torch.cuda.synchronize()
    clk.__exit__(None, None, None)
    _trace("main measurement done")
    # fixed-config strong scaling (configs[4], BH 16M): the same workload at
    # every N, so the driver's 1/2/4/8-GPU lines are comparable
    strong = strong_knn = None
    if args.workload == "bh" and not args.no_strong and not args.unsorted:
        del q_all, out, out_shard
        torch.cuda.empty_cache()
        strong = run_strong16m(args, rank, world, device, P, PAR, "bh")
        torch.cuda.empty_cache()
        strong_knn = run_strong16m(args, rank, world, device, P, PAR, "knn")
    if rank != 0:
        return
    peaks, peak_src = measured_peaks()
    hbm = float(peaks.get("hbm_gbs", 6650.0))
    bpv = BYTES_PER_VISIT[name]
    bpt = BYTES_PER_POINT_TEST.get(name, 0)
    # SURVEY §8(d) algorithmic bytes per launch on rank 0
    alg_bytes = visits * bpv + ptests * bpt + m * BYTES_PER_POINT_IO[name]
    achieved = alg_bytes / (kms / 1e3) / 1e9
    kernel_name = {"bh": "bh_group_kernel", "pc": "pc_kernel", "knn": "knn_kernel", "vp": "vp_kernel", "nn": "nn_kernel"}[name]
    if name == "pc" and args.mode == "auto" and args.variant == "autoropes" and args.auto_min_depth is None \
            and -(-m // 32) < torch.cuda.get_device_properties(device).multi_processor_count * 32:
        kernel_name = "pc_split_kernel"  # AUTO splits small launches over 16 lanes per point (tt.h)
    cnt = load_counts(args.workload, args.mode) if not args.unsorted and args.variant == "autoropes" else None
    cnt_ok = bool(cnt) and cnt.get("src_sha256") == kernel_sha256(name)
    clocks = clk.summary()
    sm_mhz = clocks.get("sm_mhz") or float(peaks.get("sm_max_mhz", 1965.0))
    nsm = torch.cuda.get_device_properties(device).multi_processor_count
    # Three views of the dominant kernel, all measured live except the ncu
    # instruction count:
    #  * `roofline` (primary): executed warp instructions / s against the
    #    issue ceiling 148 SMs x 4 schedulers x clock -- the binding roof
    #    (ncu issue slots 73-79% busy; DRAM < 2% of peak);
    #  * `hbm_effective`: SURVEY §8(d)'s algorithmic bytes / kernel time vs
    #    the measured HBM copy bandwidth (the north_star's "effective
    #    node-fetch bandwidth"); above 1 because warp fetches are broadcast
    #    to the lanes and served from L1/L2, so it is NOT HBM evidence;
    #  * `node_fetch`: bytes of the node records the warps actually fetch
    #    (warp fetches x the layout's bytes per fetched node) / kernel time,
    #    against the measured HBM bandwidth and a live L2 read ceiling
    #    (tt_diag_l2read); `traffic` = ncu DRAM bytes of the same launch.
    hbm_eff = {"bound": "hbm", "achieved": round(achieved, 1), "peak": hbm, "unit": "GB/s",
               "frac": round(achieved / hbm, 4), "peak_source": peak_src,
               "alg_bytes_per_launch": int(alg_bytes),
               "alg_bytes_def": f"useful visits x {bpv} B" + (f" + leaf-point tests x {bpt} B" if bpt else "")
                                + f" + {BYTES_PER_POINT_IO[name]} B/point I/O (SURVEY 8(d)); "
                                "served by L1/L2 and warp broadcast, not HBM"}
    fetch_bytes = wf * FETCH_BYTES[name]
    nf_gbs = fetch_bytes / (kms / 1e3) / 1e9
    node_fetch = {"achieved": round(nf_gbs, 1), "unit": "GB/s", "fetch_bytes_per_launch": int(fetch_bytes),
                  "def": f"warp node fetches (tt_stats) x {FETCH_BYTES[name]} B per fetched node of the packed "
                         "layout / kernel time",
                  "hbm_peak": hbm, "hbm_frac": round(nf_gbs / hbm, 4), "hbm_peak_source": peak_src}
    if not args.no_chase:
        l2 = l2_ceiling(P, device)
        node_fetch.update({"l2_peak": round(l2, 1), "l2_frac": round(nf_gbs / l2, 4),
                           "l2_peak_def": "tt_diag_l2read: 64 MiB L2-resident buffer, ld.global.cg, measured live"})
    common = {"kernel": kernel_name, "kernel_ms": round(kms, 4),
              "kernel_share_of_step": round(kms / ms, 4) if world == 1 else None,
              "traffic": int(cnt["dram_bytes_per_point"] * m) if cnt_ok else None,
              "traffic_def": "ncu dram__bytes_read.sum + dram__bytes_write.sum of this launch configuration"}
    if cnt_ok:
        inst = cnt["warp_inst_per_point"] * m
        issue_peak = nsm * 4 * sm_mhz * 1e6 / 1e9  # warp instructions per ns -> G/s
        roofline = {"bound": "alu", "roof": "warp-instruction issue (ALU, LSU and branch instructions all issue here)",
                    "achieved": round(inst / (kms / 1e3) / 1e9, 1), "peak": round(issue_peak, 1),
                    "unit": "Gwarp-inst/s", "frac": round(inst / (kms / 1e3) / 1e9 / issue_peak, 4),
                    "inst_per_launch": int(inst),
                    "achieved_def": f"ncu smsp__inst_executed of this kernel source and workload "
                                    f"({args.workload}, {cnt['round']}) / live kernel time",
                    "peak_def": f"{nsm} SMs x 4 schedulers x 1 warp-inst/clk x {sm_mhz:.0f} MHz (B200_PROFILING)",
                    **common, "hbm_effective": hbm_eff, "node_fetch": node_fetch}
    else:
        roofline = {**hbm_eff, **common, "issue": None, "node_fetch": node_fetch,
                    "note": "no ncu instruction count for this kernel source / workload: HBM-effective roofline only"}
    # L2-latency roof (live): a lockstep step is one 32-B record load whose
    # address comes from the previous record; tt_diag_chase runs that pure
    # dependent chase over as many records as the tree has nodes, with the
    # traversal kernels' launch shape.  Independent-mode launches compare
    # lane visits with the per-lane chase.
    if args.variant == "autoropes" and not args.no_chase:
        per_lane = lock_frac < 0.5
        peak_steps = chase_ceiling(P, tree.n_nodes, device, per_lane)
        ach = (visits if per_lane else wf) / (kms / 1e3)
        roofline["chase"] = {
            "bound": "l2-latency", "achieved": round(ach / 1e9, 3), "peak": round(peak_steps / 1e9, 3),
            "unit": "G dependent record loads/s", "frac": round(ach / peak_steps, 4),
            "achieved_def": ("lane visits" if per_lane else "lockstep warp fetches (tt_stats)") + " / kernel time",
            "peak_def": f"tt_diag_chase over {tree.n_nodes} random-cycle 32-B records, "
                        + ("one chain per lane" if per_lane else "one chain per warp (uniform loads)")
                        + ", 4 x 256-thread CTAs per SM, measured live"}
    cpu = None
    if world == 1 and not args.no_cpu_baseline:
        try:
            cpu = oracle_baseline(name, w)
        except Exception as e:  # noqa: BLE001
            cpu = {"value": None, "error": repr(e)}
    value = n_all / (ms / 1e3)  # all points of all ranks per second
    line = {
        "metric": METRIC, "value": value, "unit": "points/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": "strong" if w.get("strong") else "weak",
        "vs_baseline": None, "dtype": "f32", "data": "synthetic",
        "config": {"workload": w["workload"], "points_per_rank": m, "global_points": n_all,
                   "tree_points": w["n_data"], "mode": args.mode, "sorted": not args.unsorted,
                   "tile_schedule": "longest-first" if lpt else "in-order",
                   **({"switch_below": args.switch_below} if args.switch_below else {}),
                   "auto_min_depth": args.auto_min_depth, "variant": args.variant,
                   "parallelism": f"dp{world} (points sharded by global tree order, tree replicated)"
                   if world > 1 and not args.unsorted else f"dp{world} (points sharded, tree replicated)",
                   "l2": "flushed between timed steps (256 MiB write, 2x L2)",
                   "params": {k: v for k, v in c.items() if k not in ("kind",)}},
        "node_visits_per_sec": visits_tot / (kms / 1e3),
        "visits_per_point": visits / m,
        "lockstep_warp_fraction": lock_frac,
        # lane-slots offered by the warp fetches / useful visits (lockstep tiles)
        "work_expansion_fetch_over_visits": (wf * tile_pts / visits)
        if visits and lock_frac > 0.99 else None,
        "work_expansion_table2": we_table2,
        "warp_tile_points": tile_pts,
        "traverse_ms": kms, "upload_ms": upload_ms, "tree_build_ms": build_ms, "tree_build": build_where,
        "group_build_ms": group_build_ms, "bcast_ms": bcast_ms, "placement_ms": placement_ms,
        "allgather_ms": allgather_ms,
        "roofline": roofline, "cpu_baseline": cpu, "e2e": e2e, "strong_16m": strong, "strong_16m_knn": strong_knn,
        "paper_context": PAPER_CONTEXT.get(name),
        "gpu_launches": (launches or 0) * args.steps,
        "gpu_launches_per_step": launches,
        "clocks": clocks,
    }
    print(json.dumps(line), flush=True)


def main():
    args = parse()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        if world == 1 and args.gpus > 1:
            print(json.dumps({"error": "launch N>1 under torchrun"}), flush=True)
            sys.exit(2)
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        backend = os.environ.get("TT_DIST_BACKEND", "nccl")  # gloo: multi-rank flow test on one GPU
        if backend == "gloo":
            os.environ.setdefault("GLOO_SOCKET_IFNAME", "lo")  # loopback: the hostname may not resolve
        gpu = local_rank % torch.cuda.device_count()
        torch.cuda.set_device(gpu)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", gpu))
        else:
            dist.init_process_group(backend)
    try:
        if args.workload == "bhsteps":
            run_bh_steps(args, rank, world)
        else:
            run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()

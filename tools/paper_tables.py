"""Table 1 / Table 2 of the paper re-measured on
B200 with this repo's kernels and synthetic inputs (context, not parity).

  python tools/paper_tables.py [--out gpurun_out/paper_tables.md]

Per benchmark (BH, PC, kNN, NN, VP at the BASELINE configs; NN on configs[2]'s
inputs), per order (sorted = tt_sort_points, unsorted = input order) and mode
(L = lockstep, N = independent autoropes):
  * traversal time (CUDA events on the launch stream, median of 3 after 2
    warm-ups);
  * avg # nodes = truncation tests per point (the paper's per-point count,
    P:L1236-1240; for L the tests a lane takes while in the warp mask);
  * work expansion (Table 2, L only) = mean over warp tiles of
    warp node fetches / longest lane's visits (reading R15);
  * speedup vs the oracle on 1 and on all host cores (the paper's "vs 1" /
    "vs 32" columns used a 32-thread Opteron; the oracle is a plain recursive
    C program, not a tuned CPU code), timed on a bounded sample;
  * improvement vs the naive recursive GPU kernel (TT_VARIANT_RECURSIVE, N).
"""
from __future__ import annotations

import argparse
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402
import oracle  # noqa: E402
import paper_conf_sc_goldfarbjk13_b200 as P  # noqa: E402


def timed(fn, reps=3, warm=2):
    s = torch.cuda.current_stream()
    for _ in range(warm):
        fn()
    ts = []
    for _ in range(reps):
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        fn()
        b.record(s)
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b))
    return statistics.median(ts)


def oracle_rate(name, w, threads, seconds_target=3.0):
    """points/s of the oracle on `threads` host threads over a growing sample."""
    c, q = w["cfg"], w["queries"]
    tree = {"bh": lambda: oracle.build_oct(w["data"]), "vp": lambda: oracle.build_vp(w["data"]),
            "nn": lambda: oracle.build_nn(w["data"])}.get(name, lambda: oracle.build_kd(w["data"], c["leaf"]))()
    run = {"bh": lambda s: oracle.bh(tree, q[s], c["theta"], c["eps"], self_ids=s, threads=threads),
           "pc": lambda s: oracle.pc(tree, q[s], c["radius"], threads=threads),
           "knn": lambda s: oracle.knn(tree, q[s], c["k"], threads=threads),
           "vp": lambda s: oracle.vp(tree, q[s], threads=threads),
           "nn": lambda s: oracle.nn(tree, q[s], threads=threads)}[name]
    m = 64
    while True:
        sel = np.linspace(0, len(q) - 1, min(m, len(q))).astype(np.int64)
        t0 = time.perf_counter()
        run(sel)
        dt = time.perf_counter() - t0
        if dt >= seconds_target or m >= len(q):
            return len(sel) / dt
        m = int(m * min(8.0, max(2.0, seconds_target / max(dt, 1e-3))))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "paper_tables.md"))
    ap.add_argument("--cpu-seconds", type=float, default=3.0)
    args = ap.parse_args()
    dev = torch.device("cuda:0")
    ncpu = oracle.max_threads()
    rows = []
    for name in ("bh", "pc", "knn", "nn", "vp"):
        w = bench.make_workload(name, 1)
        c = w["cfg"]
        tree = P.tt_tree_upload(bench.host_tree(P, name, w))
        q = torch.from_numpy(np.ascontiguousarray(w["queries"][: w["m"]])).to(dev)
        m = q.shape[0]
        T = P._lib.TILE_POINTS[tree.kind]

        def launch(order, mode, stats=None, variant="autoropes"):
            if name == "bh":
                return P.tt_traverse_bh(tree, q, c["theta"], c["eps"], order=order, mode=mode, stats=stats,
                                        variant=variant)
            if name == "pc":
                return P.tt_traverse_pc(tree, q, c["radius"], order=order, mode=mode, stats=stats, variant=variant)
            if name == "knn":
                return P.tt_traverse_knn(tree, q, c["k"], order=order, mode=mode, stats=stats, variant=variant)
            if name == "vp":
                return P.tt_traverse_vp(tree, q, order=order, mode=mode, stats=stats, variant=variant)
            return P.tt_traverse_nn(tree, q, order=order, mode=mode, stats=stats)

        rate1 = oracle_rate(name, w, 1, args.cpu_seconds)
        rateN = oracle_rate(name, w, ncpu, args.cpu_seconds)
        sorted_order = P.tt_sort_points(tree, q)
        rec_ms = None
        if name != "nn":
            rec_ms = timed(lambda: launch(sorted_order, "independent", variant="recursive"), reps=1, warm=1)
        for oname, order in (("sorted", sorted_order), ("unsorted", None)):
            vis_n = None
            for mode in ("independent", "lockstep"):
                ms = timed(lambda: launch(order, mode))
                st = P.Stats.alloc(m, dev)
                launch(order, mode, stats=st)
                torch.cuda.synchronize()
                vis = st.visits.to(torch.int64).cpu().numpy()
                nodes = vis.mean()
                we = None
                if mode == "independent":
                    vis_n = vis
                else:
                    # Table 2: nodes the lockstep warp tests /
                    # nodes of its longest non-lockstep traversal (N-mode
                    # visits of the same points), per warp tile of T points
                    o = sorted_order.cpu().numpy() if order is not None else np.arange(m)
                    v = vis_n[o]
                    nt = m // T
                    longest = v[: nt * T].reshape(nt, T).max(1)
                    wt = st.warp_steps[:nt].to(torch.int64).cpu().numpy()
                    we = float(np.mean(wt / np.maximum(longest, 1)))
                pts_s = m / (ms / 1e3)
                rows.append(dict(bench=name, workload=w["workload"], order=oname, mode="L" if mode == "lockstep" else "N",
                                 ms=ms, nodes=nodes, we=we, vs1=pts_s / rate1, vsN=pts_s / rateN,
                                 rec=(rec_ms / ms) if (rec_ms and mode == "independent" and oname == "sorted") else None))
        print(name, "done", flush=True)

    lines = ["# Table 1 / Table 2 analogue on B200 (tools/paper_tables.py)", "",
             f"Host oracle threads: {ncpu} (`vs all`), 1 (`vs 1`); the paper's CPU columns used a 32-thread "
             "Opteron and a C2070 GPU (P:L1110-1117), context only.  L = lockstep, N = independent; "
             "avg # nodes = truncation tests per point; work expansion = mean over warp tiles of "
             "nodes the lockstep warp tests / the longest independent traversal among its points "
             "(Table 2, P:L2307-2313; BH tiles hold 64 bodies, the others 32); improv. vs recurse = naive recursive GPU kernel time / "
             "autoropes time (N, sorted).", "",
             "| benchmark | order | mode | time (ms) | avg # nodes | work expansion | speedup vs 1 | speedup vs all | improv. vs recurse |",
             "|---|---|---|---|---|---|---|---|---|"]
    for r in rows:
        we = "" if r["we"] is None else f"{r['we']:.2f}"
        rec = "" if r["rec"] is None else f"{r['rec']:.1f}x"
        lines.append(f"| {r['workload']} | {r['order']} | {r['mode']} | {r['ms']:.3f} | {r['nodes']:.0f} | {we} | "
                     f"{r['vs1']:.0f}x | {r['vsN']:.1f}x | {rec} |")
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    open(args.out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    main()

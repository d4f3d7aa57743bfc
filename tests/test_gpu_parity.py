"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle on the
same seeded inputs.  Bars:
  * PC counts, kNN / VP indices and d2, sort permutations, per-point visit
    counts: bit-exact;
  * BH accelerations: max_i |a_gpu - a_ref| / |a_ref| <= 1e-4 against the fp64
    oracle (north_star), with opening decisions pinned (visit counts exact).
Sizes span many warp tiles and a ragged tail; config-sized cases check
sampled outputs the oracle computes one by one.
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import ttgen

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_sc_goldfarbjk13_b200 as P

MODES = ["lockstep", "independent", "auto"]
BH_TOL = 1e-4


def dev(a, dtype=torch.float32):
    return torch.from_numpy(np.ascontiguousarray(a)).to("cuda", dtype)


def perm_i32(p):
    return dev(p.astype(np.int32), torch.int32)


def rel_err(a_gpu, a_ref):
    return np.linalg.norm(a_gpu[:, :3].astype(np.float64) - a_ref, axis=1) / np.linalg.norm(a_ref, axis=1)


# ---------------------------------------------------------------- PC (config 1)
@pytest.fixture(scope="module")
def pc_setup():
    c = ttgen.CONFIGS["pc_10k_3d"]
    p = ttgen.uniform(c["n"], c["dim"], c["seed"])
    ot = oracle.build_kd(p, c["leaf"])
    ref = oracle.pc(ot, p, c["radius"], stats=True)
    tree = P.tt_tree_upload(P.build_kd(p, c["leaf"]))
    return c, p, ot, ref, tree


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("sorted_", [False, True])
def test_pc_config1_bit_exact(pc_setup, mode, sorted_):
    c, p, ot, ref, tree = pc_setup
    q = dev(p)
    order = P.tt_sort_points(tree, q) if sorted_ else None
    st = P.Stats.alloc(len(p), "cuda")
    cnt = P.tt_traverse_pc(tree, q, c["radius"], order=order, mode=mode, stats=st)
    torch.cuda.synchronize()
    assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), ref.out[0])
    # each lane tests exactly its own recursive visit sequence (both modes)
    assert np.array_equal(st.visits.cpu().numpy(), ref.visits)
    if mode == "lockstep":
        o = order.cpu().numpy() if sorted_ else np.arange(len(p))
        union = oracle.unguided_warp_union(ot, p[o], c["radius"])
        assert np.array_equal(st.warp_fetches.cpu().numpy(), union)


def test_pc_ragged_and_buckets():
    p = ttgen.gaussian_mixture(5000, 7, seed=201, components=6)
    q = ttgen.gaussian_mixture(1237, 7, seed=202, components=6)
    ot = oracle.build_kd(p, 8)
    ref = oracle.pc(ot, q, 0.15, stats=True)
    tree = P.tt_tree_upload(P.build_kd(p, 8))
    for mode in MODES:
        st = P.Stats.alloc(len(q), "cuda")
        cnt = P.tt_traverse_pc(tree, dev(q), 0.15, mode=mode, stats=st)
        assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), ref.out[0])
        assert np.array_equal(st.visits.cpu().numpy(), ref.visits)


# ------------------------------------------------------------------------ BH
@pytest.fixture(scope="module")
def bh_small():
    b = ttgen.plummer(20011, seed=203)
    ot = oracle.build_oct(b)
    ref = oracle.bh(ot, b, 0.5, 0.05, self_ids=np.arange(len(b)), stats=True)
    tree = P.tt_tree_upload(P.build_oct(b))
    return b, ot, ref, tree


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("sorted_", [False, True])
def test_bh_within_1e4_and_same_openings(bh_small, mode, sorted_):
    b, ot, ref, tree = bh_small
    bd = dev(b)
    order = P.tt_sort_points(tree, bd) if sorted_ else None
    st = P.Stats.alloc(len(b), "cuda")
    acc = P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=order, mode=mode, stats=st).cpu().numpy()
    err = rel_err(acc, ref.out[0])
    assert err.max() <= BH_TOL, err.max()
    assert np.array_equal(st.visits.cpu().numpy(), ref.visits)
    assert np.all(acc[:, 3] == 0)
    if mode == "lockstep":
        # a BH warp tile holds 64 bodies (2 per lane): its fetches are the union
        # of 64 traversals
        o = order.cpu().numpy() if sorted_ else np.arange(len(b))
        W = 32 * P._lib.BH_POINTS_PER_LANE  # a BH warp tile holds 64 bodies
        union = oracle.unguided_warp_union(ot, b[o], 0.5, W=W)
        assert np.array_equal(st.warp_fetches.cpu().numpy()[:len(union)], union)


def test_bh_lockstep_equals_independent(bh_small):
    """Default BH path: each body makes the same opening decisions in both
    modes (identical visit counts); the child-group lockstep walk adds the
    body's terms in DFS-over-groups order (reading R23), so L and N agree to
    rounding.  (The per-node lockstep walks are bit-identical to N:
    tests/test_gpu_order.py.)"""
    b, ot, ref, tree = bh_small
    bd = dev(b)
    sl, sn = P.Stats.alloc(len(b), "cuda"), P.Stats.alloc(len(b), "cuda")
    a_l = P.tt_traverse_bh(tree, bd, 0.5, 0.05, mode="lockstep", stats=sl).cpu().numpy()
    a_n = P.tt_traverse_bh(tree, bd, 0.5, 0.05, mode="independent", stats=sn).cpu().numpy()
    assert np.array_equal(sl.visits.cpu().numpy(), sn.visits.cpu().numpy())
    assert rel_err(a_l, a_n[:, :3].astype(np.float64)).max() < 2e-6


def test_bh_theta0_direct_sum_and_duplicates():
    from tests import brute
    b = ttgen.plummer(3001, seed=204)
    b[100, :3] = b[101, :3] = b[102, :3]
    tree = P.tt_tree_upload(P.build_oct(b))
    acc = P.tt_traverse_bh(tree, dev(b), 0.0, 0.05).cpu().numpy()
    err = rel_err(acc, brute.direct_sum(b, 0.05))
    assert err.max() <= BH_TOL


@pytest.mark.slow
def test_bh_config2_full_size_sampled():
    c = ttgen.CONFIGS["bh_1m_plummer"]
    b = ttgen.plummer(c["n"], c["seed"])
    ot = oracle.build_oct(b)
    tree = P.tt_tree_upload(P.build_oct(b))
    bd = dev(b)
    perm = P.tt_sort_points(tree, bd)
    st = P.Stats.alloc(len(b), "cuda")
    acc = P.tt_traverse_bh(tree, bd, c["theta"], c["eps"], order=perm, stats=st).cpu().numpy()
    rng = np.random.default_rng(0)
    sample = np.concatenate([rng.choice(len(b), 20000, replace=False),
                             np.argsort(np.linalg.norm(b[:, :3], axis=1))[:2000]])  # incl. the core
    ref = oracle.bh(ot, b[sample], c["theta"], c["eps"], self_ids=sample, stats=True)
    err = rel_err(acc[sample], ref.out[0])
    w = int(np.argmax(err))
    print(f"BH 1M sampled: max rel err {err.max():.3e} at body {sample[w]} "
          f"(r={np.linalg.norm(b[sample[w], :3]):.4f}), p99.99 {np.quantile(err, 0.9999):.3e}")
    assert err.max() <= BH_TOL, err.max()
    assert np.array_equal(st.visits.cpu().numpy()[sample], ref.visits)


# ----------------------------------------------------------------------- kNN
@pytest.fixture(scope="module")
def knn_small():
    p = ttgen.gaussian_mixture(20000, 7, seed=205, components=12)
    p[500:510] = p[3]
    q = np.concatenate([ttgen.gaussian_mixture(4990, 7, seed=206, components=12), p[:21]])
    ot = oracle.build_kd(p, 8)
    tree = P.tt_tree_upload(P.build_kd(p, 8))
    return p, q, ot, tree


@pytest.mark.parametrize("k", [1, 8, 13, 32])
def test_knn_independent_bit_exact(knn_small, k):
    p, q, ot, tree = knn_small
    ref = oracle.knn(ot, q, k, stats=True)
    st = P.Stats.alloc(len(q), "cuda")
    idx, d2 = P.tt_traverse_knn(tree, dev(q), k, mode="independent", stats=st)
    assert np.array_equal(idx.cpu().numpy(), ref.out[0])
    assert np.array_equal(d2.cpu().numpy(), ref.out[1])
    assert np.array_equal(st.visits.cpu().numpy(), ref.visits)  # same order => same pruning


@pytest.mark.parametrize("sorted_", [False, True])
def test_knn_lockstep_matches_fig8_simulation(knn_small, sorted_):
    p, q, ot, tree = knn_small
    qd = dev(q)
    order = P.tt_sort_points(tree, qd) if sorted_ else None
    o = order.cpu().numpy() if sorted_ else np.arange(len(q))
    li, ld, lv, wf = oracle.knn_lockstep(ot, q[o], 8)
    st = P.Stats.alloc(len(q), "cuda")
    idx, d2 = P.tt_traverse_knn(tree, qd, 8, order=order, mode="lockstep", stats=st)
    ref = oracle.knn(ot, q, 8)
    assert np.array_equal(idx.cpu().numpy(), ref.out[0]) and np.array_equal(d2.cpu().numpy(), ref.out[1])
    assert np.array_equal(st.visits.cpu().numpy()[o], lv)
    assert np.array_equal(st.warp_fetches.cpu().numpy(), wf)


def test_knn_pads_when_k_exceeds_points():
    p = ttgen.uniform(5, 3, seed=207)
    tree = P.tt_tree_upload(P.build_kd(p, 2))
    ref = oracle.knn(oracle.build_kd(p, 2), p, 8)
    for mode in MODES:
        idx, d2 = P.tt_traverse_knn(tree, dev(p), 8, mode=mode)
        assert np.array_equal(idx.cpu().numpy(), ref.out[0]) and np.array_equal(d2.cpu().numpy(), ref.out[1])


@pytest.mark.slow
def test_knn_config3_full_size_sampled():
    c = ttgen.CONFIGS["knn_1m_7d"]
    p = ttgen.gaussian_mixture(c["n"], c["dim"], c["seed"])
    q = ttgen.gaussian_mixture(c["m"], c["dim"], c["qseed"])
    ot = oracle.build_kd(p, c["leaf"])
    tree = P.tt_tree_upload(P.build_kd(p, c["leaf"]))
    qd = dev(q)
    perm = P.tt_sort_points(tree, qd)
    idx, d2 = P.tt_traverse_knn(tree, qd, c["k"], order=perm)
    sample = np.random.default_rng(1).choice(len(q), 3000, replace=False)
    ref = oracle.knn(ot, q[sample], c["k"])
    assert np.array_equal(idx.cpu().numpy()[sample], ref.out[0])
    assert np.array_equal(d2.cpu().numpy()[sample], ref.out[1])


# ------------------------------------------------------------------------ VP
@pytest.fixture(scope="module")
def vp_small():
    p = ttgen.gaussian_mixture(20000, 16, seed=208, components=10)
    p[700:704] = p[9]
    q = np.concatenate([ttgen.gaussian_mixture(3000, 16, seed=209, components=10), p[:13]])
    ot = oracle.build_vp(p)
    tree = P.tt_tree_upload(P.build_vp(p))
    return p, q, ot, tree


def test_vp_independent_bit_exact(vp_small):
    p, q, ot, tree = vp_small
    ref = oracle.vp(ot, q, stats=True)
    st = P.Stats.alloc(len(q), "cuda")
    idx, d2 = P.tt_traverse_vp(tree, dev(q), mode="independent", stats=st)
    assert np.array_equal(idx.cpu().numpy(), ref.out[0])
    assert np.array_equal(d2.cpu().numpy(), ref.out[1])
    assert np.array_equal(st.visits.cpu().numpy(), ref.visits)


@pytest.mark.parametrize("sorted_", [False, True])
def test_vp_lockstep_matches_simulation(vp_small, sorted_):
    p, q, ot, tree = vp_small
    qd = dev(q)
    order = P.tt_sort_points(tree, qd) if sorted_ else None
    o = order.cpu().numpy() if sorted_ else np.arange(len(q))
    li, ld, lv, wf = oracle.vp_lockstep(ot, q[o])
    st = P.Stats.alloc(len(q), "cuda")
    idx, d2 = P.tt_traverse_vp(tree, qd, order=order, mode="lockstep", stats=st)
    assert np.array_equal(idx.cpu().numpy()[o], li) and np.array_equal(d2.cpu().numpy()[o], ld)
    assert np.array_equal(st.visits.cpu().numpy()[o], lv)
    assert np.array_equal(st.warp_fetches.cpu().numpy(), wf)


def test_vp_auto_results_exact(vp_small):
    p, q, ot, tree = vp_small
    ref = oracle.vp(ot, q)
    qd = dev(q)
    for sorted_ in (False, True):
        order = P.tt_sort_points(tree, qd) if sorted_ else None
        idx, d2 = P.tt_traverse_vp(tree, qd, order=order, mode="auto")
        assert np.array_equal(idx.cpu().numpy(), ref.out[0]) and np.array_equal(d2.cpu().numpy(), ref.out[1])


@pytest.mark.slow
def test_vp_config4_full_size_sampled():
    c = ttgen.CONFIGS["vp_1m_16d"]
    p = ttgen.gaussian_mixture(c["n"], c["dim"], c["seed"])
    q = ttgen.gaussian_mixture(c["m"], c["dim"], c["qseed"])
    ot = oracle.build_vp(p)
    tree = P.tt_tree_upload(P.build_vp(p))
    qd = dev(q)
    perm = P.tt_sort_points(tree, qd)
    idx, d2 = P.tt_traverse_vp(tree, qd, order=perm)
    sample = np.random.default_rng(2).choice(len(q), 400, replace=False)
    ref = oracle.vp(ot, q[sample])
    assert np.array_equal(idx.cpu().numpy()[sample], ref.out[0])
    assert np.array_equal(d2.cpu().numpy()[sample], ref.out[1])


# ---------------------------------------------------------------------- sort
def _pinned_d2(q, p):
    """fp32 sequential squared distance, one rounding per operation (R0)."""
    t = (q[..., 0] - p[..., 0]).astype(np.float32)
    s = (t * t).astype(np.float32)
    for d in range(1, q.shape[-1]):
        t = (q[..., d] - p[..., d]).astype(np.float32)
        s = (s + (t * t).astype(np.float32)).astype(np.float32)
    return s


def _tiles(a, T):
    nfull = len(a) // T
    return [tuple(a[i * T:(i + 1) * T]) for i in range(nfull)], a[nfull * T:]


def _check_tile_permutation(perm, sched, T):
    tp, tail_p = _tiles(perm, T)
    ts, tail_s = _tiles(sched, T)
    assert np.array_equal(tail_p, tail_s)  # ragged last tile stays last
    assert sorted(tp) == sorted(ts)        # whole tiles move, contents untouched
    return tp, ts


def test_schedule_tiles_kd_longest_first(knn_small):
    """a1b on a kd tree: whole tiles reordered by the estimate recomputed here
    (leaf by the split rule, largest pinned d2 to its points), non-increasing,
    ties in point-sort order."""
    p, q, ot, tree = knn_small
    qd = dev(q)
    perm = P.tt_sort_points(tree, qd)
    sched = P.tt_schedule_tiles(tree, qd, perm).cpu().numpy()
    perm = perm.cpu().numpy()
    tp, ts = _check_tile_permutation(perm, sched, 32)
    sd, sp = ot.i64(oracle.F_SPLITDIM), ot.f32(oracle.F_SPLIT)
    ch, pb, pc = ot.children(), ot.i64(oracle.F_PBEGIN), ot.i64(oracle.F_PCOUNT)
    tpts = p[ot.tree_order()]
    cur = np.zeros(len(q), np.int64)
    for _ in range(ot.height + 1):
        inner = ch[cur, 0] >= 0
        x = q[np.arange(len(q)), np.maximum(sd[cur], 0)]
        cur = np.where(inner, np.where(x < sp[cur], ch[cur, 0], ch[cur, 1]), cur)
    est = np.zeros(len(q), np.float32)
    for j in range(int(pc.max())):
        has = j < pc[cur]
        d2 = _pinned_d2(q, tpts[pb[cur] + np.minimum(j, pc[cur] - 1)])
        est = np.where(has, np.maximum(est, d2), est)
    key = {t: est[list(t)].max() for t in tp}
    ks = np.array([key[t] for t in ts])
    assert np.all(ks[:-1] >= ks[1:])
    pos = {t: i for i, t in enumerate(tp)}
    for a, b in zip(ts[:-1], ts[1:]):  # stable among equal estimates
        if key[a] == key[b]:
            assert pos[a] < pos[b]


def test_schedule_tiles_results_unchanged(knn_small, vp_small):
    """Traversal results do not depend on the tile schedule (kNN, VP; in-place
    call; oct trees get a copy)."""
    p, q, ot, tree = knn_small
    qd = dev(q)
    perm = P.tt_sort_points(tree, qd)
    sched = P.tt_schedule_tiles(tree, qd, perm.clone())
    again = perm.clone()
    P.tt_schedule_tiles(tree, qd, again, out=again)
    assert torch.equal(sched, again)
    assert not torch.equal(sched, perm)
    for mode in MODES:
        a = P.tt_traverse_knn(tree, qd, 8, order=perm, mode=mode)
        b = P.tt_traverse_knn(tree, qd, 8, order=sched, mode=mode)
        assert torch.equal(a[0], b[0]) and torch.equal(a[1], b[1])
    p, q, ot, tree = vp_small
    qd = dev(q)
    perm = P.tt_sort_points(tree, qd)
    sched = P.tt_schedule_tiles(tree, qd, perm)
    _check_tile_permutation(perm.cpu().numpy(), sched.cpu().numpy(), 32)
    for mode in MODES:
        a = P.tt_traverse_vp(tree, qd, order=perm, mode=mode)
        b = P.tt_traverse_vp(tree, qd, order=sched, mode=mode)
        assert torch.equal(a[0], b[0]) and torch.equal(a[1], b[1])
    b = ttgen.plummer(3000, seed=214)
    t_oct = P.tt_tree_upload(P.build_oct(b))
    bd = dev(b)
    perm = P.tt_sort_points(t_oct, bd)
    assert torch.equal(P.tt_schedule_tiles(t_oct, bd, perm), perm)


def test_sort_points_matches_oracle_for_every_kind():
    b = ttgen.plummer(30000, seed=210)
    p7 = ttgen.gaussian_mixture(30000, 7, seed=211, components=8)
    q7 = ttgen.gaussian_mixture(7777, 7, seed=212, components=8)
    p16 = ttgen.gaussian_mixture(8000, 16, seed=213, components=8)
    cases = [(P.build_oct(b), oracle.build_oct(b), b),
             (P.build_kd(p7, 8), oracle.build_kd(p7, 8), q7),
             (P.build_vp(p16), oracle.build_vp(p16), p16)]
    for host, ot, pts in cases:
        tree = P.tt_tree_upload(host)
        keys = torch.empty(len(pts), dtype=torch.int64, device="cuda")
        perm = P.tt_sort_points(tree, dev(pts), keys=keys)
        assert np.array_equal(keys.cpu().numpy().view(np.uint64), oracle.sort_keys(ot, pts))
        assert np.array_equal(perm.cpu().numpy(), oracle.sort_perm(ot, pts))


@pytest.mark.parametrize("n", [1, 33, 16384, 16385])
def test_kd_sort_sizes_with_equal_keys(n):
    """kd sorts from one point to past 2^14 points (a one-CTA shared-memory
    sort for <= 16384 points was tried there and measured no faster, DESIGN
    §4.6) equal the oracle's stable (key, index) order, with many equal keys
    (leaf 8)."""
    p = ttgen.gaussian_mixture(20000, 3, seed=215, components=6)
    host, ot = P.build_kd(p, 8), oracle.build_kd(p, 8)
    tree = P.tt_tree_upload(host)
    q = np.ascontiguousarray(p[np.random.default_rng(n).integers(0, len(p), n)])
    perm = P.tt_sort_points(tree, dev(q))
    assert np.array_equal(perm.cpu().numpy(), oracle.sort_perm(ot, q))


# ------------------------------------------------------------ edges / misc
def test_empty_and_partial_warp():
    p = ttgen.uniform(1000, 3, seed=214)
    tree = P.tt_tree_upload(P.build_kd(p, 1))
    ot = oracle.build_kd(p, 1)
    out = P.tt_traverse_pc(tree, dev(p[:0]), 0.1)
    assert out.numel() == 0
    for n in (1, 7, 31, 33):
        for mode in MODES:
            cnt = P.tt_traverse_pc(tree, dev(p[:n]), 0.2, mode=mode).cpu().numpy()
            assert np.array_equal(cnt.astype(np.uint32), oracle.pc(ot, p[:n], 0.2).out[0])


def test_kind_mismatch_is_reported():
    p = ttgen.uniform(100, 3, seed=215)
    tree = P.tt_tree_upload(P.build_kd(p, 1))
    with pytest.raises(P.TTError) as e:
        P.tt_traverse_bh(tree, dev(np.zeros((4, 4), np.float32)), 0.5, 0.05)
    assert e.value.status == -5


def test_sharded_launches_concatenate_to_full_run(bh_small):
    """Multi-GPU invariant simulated on one GPU: G warp-aligned contiguous
    slices of the sorted order (parallel.shard_range), run one after another,
    equal the single run bit for bit."""
    from paper_conf_sc_goldfarbjk13_b200.parallel import shard_range
    b, ot, ref, tree = bh_small
    bd = dev(b)
    perm = P.tt_sort_points(tree, bd)
    full = P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=perm).cpu().numpy()
    out = torch.zeros((len(b), 4), device="cuda")
    G = 4
    for g in range(G):
        lo, hi = shard_range(len(b), g, G)
        P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=perm[lo:hi].contiguous(), out=out)
    assert np.array_equal(out.cpu().numpy(), full)


def test_blob_roundtrip_device_adoption():
    """tt_tree_from_blob(mem=DEVICE): the NCCL-broadcast path."""
    b = ttgen.plummer(5000, seed=216)
    host = P.build_oct(b)
    blob = torch.from_numpy(host.pack()).cuda()
    t1 = P.tt_tree_upload(host)
    t2 = P.tt_tree_from_blob(blob)
    bd = dev(b)
    a1 = P.tt_traverse_bh(t1, bd, 0.5, 0.05).cpu().numpy()
    a2 = P.tt_traverse_bh(t2, bd, 0.5, 0.05).cpu().numpy()
    assert np.array_equal(a1, a2)


@pytest.mark.slow
def test_bh_config5_16m_sampled():
    """configs[4]: 16,777,216-body Plummer sphere (the multi-GPU config) on one
    GPU, sampled bodies against the oracle."""
    c = ttgen.CONFIGS["bh_16m_plummer"]
    b = ttgen.plummer(c["n"], c["seed"])
    tree = P.tt_tree_upload(P.build_oct(b))
    bd = dev(b)
    perm = P.tt_sort_points(tree, bd)
    acc = P.tt_traverse_bh(tree, bd, c["theta"], c["eps"], order=perm).cpu().numpy()
    ot = oracle.build_oct(b)
    sample = np.concatenate([np.random.default_rng(3).choice(len(b), 4000, replace=False),
                             np.argsort(np.linalg.norm(b[:, :3], axis=1))[:500]])
    ref = oracle.bh(ot, b[sample], c["theta"], c["eps"], self_ids=sample)
    err = rel_err(acc[sample], ref.out[0])
    print(f"BH 16M sampled: max rel err {err.max():.3e}")
    assert err.max() <= BH_TOL


@pytest.mark.slow
def test_knn_config5_16m_sampled():
    """configs[4]: kNN k=8, 16,777,216 queries over 16,777,216 7-D mixture
    points, in the launch configuration bench.py times (device-built tree,
    sort + longest-first schedule, AUTO); sampled queries bit-exact against
    brute force over all 16M points (the plain definition, R4)."""
    c = ttgen.CONFIGS["knn_16m_7d"]
    p = ttgen.gaussian_mixture(c["n"], c["dim"], c["seed"])
    q = ttgen.gaussian_mixture(c["m"], c["dim"], c["qseed"])
    pd, qd = dev(p), dev(q)
    tree = P.tt_build_kd_device(pd, c["leaf"])
    perm = P.tt_schedule_tiles(tree, qd, P.tt_sort_points(tree, qd))
    idx, d2 = P.tt_traverse_knn(tree, qd, c["k"], order=perm)
    sample = np.random.default_rng(4).choice(len(q), 24, replace=False)
    gi, gd = idx.cpu().numpy(), d2.cpu().numpy()
    for i in sample:
        D = _pinned_d2(q[i][None, :], p)  # the plain definition over all points
        kth = np.partition(D, c["k"] - 1)[c["k"] - 1]
        cand = np.nonzero(D <= kth)[0]
        best = cand[np.lexsort((cand, D[cand]))][: c["k"]]  # (d2, id) order
        assert np.array_equal(gi[i], best) and np.array_equal(gd[i], D[best])


# ------------------------------------------------ recursive baseline (NEXT-2)
def test_recursive_baseline_matches_oracle(bh_small, knn_small, vp_small, pc_setup):
    """The naive recursive GPU baseline computes the same results
    and visits the same nodes as the oracle -- it differs from the autoroped
    kernels only in using device recursion."""
    b, ot, ref, tree = bh_small
    acc = P.tt_traverse_bh(tree, dev(b), 0.5, 0.05, mode="independent", variant="recursive").cpu().numpy()
    assert rel_err(acc, ref.out[0]).max() <= BH_TOL
    c, p, otp, refp, treep = pc_setup
    cnt = P.tt_traverse_pc(treep, dev(p), c["radius"], mode="independent", variant="recursive")
    assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), refp.out[0])
    p, q, otk, treek = knn_small
    refk = oracle.knn(otk, q, 8)
    idx, d2 = P.tt_traverse_knn(treek, dev(q), 8, mode="independent", variant="recursive")
    assert np.array_equal(idx.cpu().numpy(), refk.out[0]) and np.array_equal(d2.cpu().numpy(), refk.out[1])
    p, q, otv, treev = vp_small
    refv = oracle.vp(otv, q, stats=True)
    idx, d2 = P.tt_traverse_vp(treev, dev(q), mode="independent", variant="recursive")
    assert np.array_equal(idx.cpu().numpy(), refv.out[0]) and np.array_equal(d2.cpu().numpy(), refv.out[1])


# ------------------------------------------------ per-warp mode choice (a2)
def test_auto_mode_choice_follows_coherence(bh_small, knn_small, vp_small):
    """AUTO (reading R19): sorted tiles run lockstep (even those straddling a
    top-level split), unsorted tiles run independent -- and results equal the
    lockstep run's (BH: up to the fp64 flush cadence)."""
    def frac(st, n, tile):  # over full tiles (a ragged last tile has few lanes to disagree)
        return (st.warp_mode.cpu().numpy()[:n // tile] == 1).mean()
    b, ot, ref, tree = bh_small
    bd = dev(b)
    for sorted_, want in ((True, 1.0), (False, 0.0)):
        order = P.tt_sort_points(tree, bd) if sorted_ else None
        st = P.Stats.alloc(len(b), "cuda")
        P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=order, stats=st)
        # 20k bodies: a few sorted tiles in the sparse outskirts span many
        # level-3 cells and count as incoherent (99.9% lockstep at 1M)
        assert abs(frac(st, len(b), 32 * P._lib.BH_POINTS_PER_LANE) - want) <= 0.03
    for (p, q, otk, treek), call in ((knn_small, lambda t, x, **kw: P.tt_traverse_knn(t, x, 8, **kw)),
                                     (vp_small, lambda t, x, **kw: P.tt_traverse_vp(t, x, **kw))):
        qd = dev(q)
        for sorted_, want in ((True, 1.0), (False, 0.0)):
            order = P.tt_sort_points(treek, qd) if sorted_ else None
            st = P.Stats.alloc(len(q), "cuda")
            idx, d2 = call(treek, qd, order=order, stats=st)
            il, dl = call(treek, qd, order=order, mode="lockstep")
            assert torch.equal(idx, il) and torch.equal(d2, dl)
            assert abs(frac(st, len(q), 32) - want) <= 0.01, (sorted_, frac(st, len(q), 32))


# ------------------------------------ explicit rope-stack variant (NEXT-3)
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("sorted_", [False, True])
def test_stack_variant_matches_oracle(bh_small, pc_setup, mode, sorted_):
    """Fig.9b's explicit rope stacks (per-thread interleaved global stacks in
    independent mode, one (node, mask) smem stack per warp in lockstep):
    same results and per-point visits as the oracle; a lockstep warp pops
    exactly the union of its 32 lanes' traversals (Fig.8)."""
    b, ot, ref, tree = bh_small
    bd = dev(b)
    order = P.tt_sort_points(tree, bd) if sorted_ else None
    st = P.Stats.alloc(len(b), "cuda")
    acc = P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=order, mode=mode, stats=st, variant="stack").cpu().numpy()
    assert rel_err(acc, ref.out[0]).max() <= BH_TOL
    assert np.array_equal(st.visits.cpu().numpy(), ref.visits)
    o = order.cpu().numpy() if sorted_ else np.arange(len(b))
    if mode != "independent":  # AUTO = lockstep for BH
        union = oracle.unguided_warp_union(ot, b[o], 0.5, W=32)
        assert np.array_equal(st.warp_fetches.cpu().numpy()[:len(union)], union)
    c, p, otp, refp, treep = pc_setup
    q = dev(p)
    order = P.tt_sort_points(treep, q) if sorted_ else None
    st = P.Stats.alloc(len(p), "cuda")
    cnt = P.tt_traverse_pc(treep, q, c["radius"], order=order, mode=mode, stats=st, variant="stack")
    assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), refp.out[0])
    assert np.array_equal(st.visits.cpu().numpy(), refp.visits)
    if mode == "lockstep":
        o = order.cpu().numpy() if sorted_ else np.arange(len(p))
        union = oracle.unguided_warp_union(otp, p[o], c["radius"])
        assert np.array_equal(st.warp_fetches.cpu().numpy(), union)


def test_stack_variant_edge_cases():
    """theta = 0 (every cell opens: the direct sum), duplicate bodies, a ragged
    last warp, buckets; kNN/VP report the variant as unsupported."""
    from tests import brute
    b = ttgen.plummer(1001, seed=240)
    b[10, :3] = b[11, :3] = b[12, :3]
    tree = P.tt_tree_upload(P.build_oct(b))
    for mode in MODES:
        acc = P.tt_traverse_bh(tree, dev(b), 0.0, 0.05, mode=mode, variant="stack").cpu().numpy()
        assert rel_err(acc, brute.direct_sum(b, 0.05)).max() <= BH_TOL
    p = ttgen.gaussian_mixture(3000, 7, seed=241, components=6)
    q = ttgen.gaussian_mixture(777, 7, seed=242, components=6)
    ot = oracle.build_kd(p, 8)
    ref = oracle.pc(ot, q, 0.15)
    t = P.tt_tree_upload(P.build_kd(p, 8))
    for mode in MODES:
        cnt = P.tt_traverse_pc(t, dev(q), 0.15, mode=mode, variant="stack")
        assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), ref.out[0])
    with pytest.raises(P.TTError):
        P.tt_traverse_knn(t, dev(q), 4, variant="stack")


# ------------------------------------------------- GPU tree build (NEXT-1)
@pytest.mark.parametrize("n,dups", [(1, False), (2, False), (3001, True), (20011, True), (1_000_000, False)])
def test_gpu_oct_build_is_byte_identical_to_host_pack(n, dups):
    """tt_build_oct_device emits exactly the blob tt_tree_pack makes from the
    host builder (itself bit-identical to the oracle's builder)."""
    b = ttgen.plummer(n, seed=217)
    if dups and n > 20:
        b[5, :3] = b[6, :3] = b[7, :3]  # depth-32 bucket
    host_blob = P.build_oct(b).pack()
    t = P.tt_build_oct_device(dev(b))
    gpu_blob = P.tt_tree_download(t)
    assert gpu_blob.size == host_blob.size
    assert np.array_equal(gpu_blob, host_blob)


# ------------------------------------------------ BH time stepping (NEXT-4)
def test_kick_drift_is_the_fp32_update():
    from paper_conf_sc_goldfarbjk13_b200 import tt_kick_drift
    rng = np.random.default_rng(5)
    x = rng.standard_normal((1000, 4)).astype(np.float32)
    v = rng.standard_normal((1000, 4)).astype(np.float32)
    a = rng.standard_normal((1000, 4)).astype(np.float32)
    X, V, A = dev(x), dev(v), dev(a)
    tt_kick_drift(X, V, A, 0.01, 0.02)
    v1 = (v[:, :3] + (a[:, :3] * np.float32(0.01)).astype(np.float32)).astype(np.float32)
    x1 = (x[:, :3] + (v1 * np.float32(0.02)).astype(np.float32)).astype(np.float32)
    assert np.array_equal(V.cpu().numpy()[:, :3], v1) and np.array_equal(X.cpu().numpy()[:, :3], x1)
    assert np.array_equal(X.cpu().numpy()[:, 3], x[:, 3])  # masses untouched


def test_two_body_circular_orbit_is_kept():
    """Physics pin of the whole time step (GPU build + sort + BH force + leapfrog):
    two equal masses on a softened circular orbit keep their separation and
    speed over a quarter orbit."""
    from paper_conf_sc_goldfarbjk13_b200 import nbody
    d, m, eps = 1.0, 0.5, 0.01
    f = m * m * d / (d * d + eps * eps) ** 1.5          # softened pair force
    vc = np.sqrt(f * (d / 2) / m)                         # m v^2 / (d/2) = f
    b = np.array([[-d / 2, 0, 0, m], [d / 2, 0, 0, m]], np.float32)
    v = np.array([[0, -vc, 0, 0], [0, vc, 0, 0]], np.float32)
    period = 2 * np.pi * (d / 2) / vc
    steps = 250
    B, V = dev(b), dev(v)
    nbody.simulate(B, V, steps, period / 4 / steps, theta=0.5, eps=eps)
    bb, vv = B.cpu().numpy().astype(np.float64), V.cpu().numpy().astype(np.float64)
    sep = np.linalg.norm(bb[1, :3] - bb[0, :3])
    assert abs(sep - d) < 1e-4
    assert np.allclose(np.linalg.norm(vv[:, :3], axis=1), vc, rtol=1e-4)
    assert np.allclose(bb[0, :3] + bb[1, :3], 0, atol=1e-5)  # centre of mass stays put
    # quarter orbit: bodies moved from the x axis to the y axis
    assert abs(bb[1, 1] - d / 2) < 1e-3 and abs(bb[1, 0]) < 1e-3


def test_plummer_steps_forces_match_oracle_each_step():
    """Five time steps of a 20k Plummer sphere: after every step the GPU force
    pass on the moved bodies matches the fp64 oracle on the same positions."""
    from paper_conf_sc_goldfarbjk13_b200 import nbody
    b = ttgen.plummer(20000, seed=218)
    v = ttgen.plummer_velocities(b, seed=219)
    B, V = dev(b), dev(v)
    acc = None
    for s in range(5):
        acc = nbody.simulate(B, V, 1, 1e-3, theta=0.5, eps=0.05, acc=acc)
        x = B.cpu().numpy()
        ref = oracle.bh(oracle.build_oct(x), x, 0.5, 0.05, self_ids=np.arange(len(x))).out[0]
        assert rel_err(acc.cpu().numpy(), ref).max() <= BH_TOL
    p = (B.cpu().numpy()[:, 3:4].astype(np.float64) * V.cpu().numpy()[:, :3]).sum(0)
    p0 = (b[:, 3:4].astype(np.float64) * v[:, :3]).sum(0)
    assert np.abs(p - p0).max() < 1e-4


@pytest.mark.parametrize("n,dim,leaf", [(1, 3, 1), (2, 3, 1), (10_000, 3, 1), (20_011, 7, 8), (5_000, 16, 4),
                                        (1_000_000, 7, 8)])
def test_gpu_kd_build_is_byte_identical_to_host_pack(n, dim, leaf):
    p = ttgen.gaussian_mixture(n, dim, seed=220, components=6)
    if n > 100:
        p[50:60] = p[7]  # duplicates: ties broken by id
    host_blob = P.build_kd(p, leaf).pack()
    t = P.tt_build_kd_device(dev(p), leaf)
    gpu_blob = P.tt_tree_download(t)
    assert gpu_blob.size == host_blob.size
    diff = np.nonzero(gpu_blob != host_blob)[0]
    assert diff.size == 0, f"{diff.size} bytes differ, first at {diff[:8]}"


@pytest.mark.parametrize("n,dim", [(1, 3), (2, 3), (3, 2), (5_000, 16), (20_011, 7), (1_000_000, 16)])
def test_gpu_vp_build_is_byte_identical_to_host_pack(n, dim):
    p = ttgen.gaussian_mixture(n, dim, seed=221, components=6)
    if n > 100:
        p[50:60] = p[7]  # equal distances: ties broken by id
    host_blob = P.build_vp(p).pack()
    t = P.tt_build_vp_device(dev(p))
    gpu_blob = P.tt_tree_download(t)
    assert gpu_blob.size == host_blob.size
    diff = np.nonzero(gpu_blob != host_blob)[0]
    assert diff.size == 0, f"{diff.size} bytes differ, first at {diff[:8]}"


# ------------------------------------------------ NEXT-3 dynamic L->N switch
@pytest.mark.parametrize("sorted_", [False, True])
def test_knn_dynamic_switch_results_exact(knn_small, sorted_):
    """Dynamic L->N switching (tt_traverse_opts.switch_below) never changes
    results; switch_below = 33 switches every tile at the root,
    so lane visits are exactly the independent walk's (autoropes order), and
    switch_below = 0 is plain lockstep (the Fig.8 simulation)."""
    p, q, ot, tree = knn_small
    qd = dev(q)
    order = P.tt_sort_points(tree, qd) if sorted_ else None
    ref = oracle.knn(ot, q, 8, stats=True)
    for a in (0, 2, 5, 12, 24, 33):
        st = P.Stats.alloc(len(q), "cuda")
        idx, d2 = P.tt_traverse_knn(tree, qd, 8, order=order, mode="lockstep", stats=st, switch_below=a)
        assert np.array_equal(idx.cpu().numpy(), ref.out[0]) and np.array_equal(d2.cpu().numpy(), ref.out[1]), a
        wm = st.warp_mode.cpu().numpy()
        if a == 33:
            assert np.all(wm == 3)
            assert np.array_equal(st.visits.cpu().numpy(), ref.visits)
        if a == 0:
            assert np.all(wm == 1)
            o = order.cpu().numpy() if sorted_ else np.arange(len(q))
            li, ld, lv, wf = oracle.knn_lockstep(ot, q[o], 8)
            assert np.array_equal(st.warp_fetches.cpu().numpy(), wf)
    with pytest.raises(P.TTError):
        P.tt_traverse_knn(tree, qd, 8, switch_below=34)


def test_diag_chase_runs_and_checks_args():
    """The roofline diagnostic (tt_diag_chase) runs in both access modes and
    rejects bad arguments; the chase records form one cycle."""
    rec = P.chase_records(1000, "cuda", seed=3)
    nxt = rec[:, 4].cpu().numpy()
    seen, cur = set(), 0
    for _ in range(1000):
        seen.add(cur)
        cur = int(nxt[cur])
    assert len(seen) == 1000 and cur == 0
    for per_lane in (False, True):
        P.tt_diag_chase(rec, 100, per_lane)
    torch.cuda.synchronize()
    with pytest.raises(P.TTError):
        P.tt_diag_chase(rec[:0], 10)


# --------------------------------------- PC traversal split over 8-lane groups
@pytest.mark.parametrize("sorted_", [False, True])
def test_pc_split_variant_exact(pc_setup, sorted_):
    """TT_VARIANT_SPLIT: every point's walk divided by subtree over 16 lanes;
    counts and per-point visit counts equal the recursive oracle's."""
    c, p, ot, ref, tree = pc_setup
    pd = dev(p)
    order = P.tt_sort_points(tree, pd) if sorted_ else None
    st = P.Stats.alloc(len(p), "cuda")
    cnt = P.tt_traverse_pc(tree, pd, c["radius"], order=order, stats=st, variant="split").cpu().numpy()
    assert np.array_equal(cnt.astype(np.uint32), ref.out[0])
    assert np.array_equal(st.visits.cpu().numpy(), ref.visits)


def test_pc_split_small_trees_and_buckets():
    for n, leaf in ((1, 1), (2, 1), (3, 1), (7, 1), (9, 2), (200, 4), (3001, 1)):
        p = ttgen.uniform(n, 3, seed=500 + n)
        q = ttgen.uniform(37, 3, seed=600 + n)
        ot = oracle.build_kd(p, leaf)
        tree = P.tt_tree_upload(P.build_kd(p, leaf))
        for r in (0.05, 0.3, 2.0):
            ref = oracle.pc(ot, q, r, stats=True)
            st = P.Stats.alloc(len(q), "cuda")
            cnt = P.tt_traverse_pc(tree, dev(q), r, stats=st, variant="split").cpu().numpy()
            assert np.array_equal(cnt.astype(np.uint32), ref.out[0]), (n, leaf, r)
            assert np.array_equal(st.visits.cpu().numpy(), ref.visits), (n, leaf, r)
    b = ttgen.plummer(100, seed=7)
    with pytest.raises(P.TTError):
        P.tt_traverse_bh(P.tt_tree_upload(P.build_oct(b)), dev(b), 0.5, 0.05, variant="split")


# ------------------------------------------- BH lockstep walk by child groups
@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("sorted_", [False, True])
def test_bh_groups_variant(bh_small, mode, sorted_):
    """TT_VARIANT_GROUPS: a lockstep warp expands whole cells; every body tests
    exactly its recursive walk's nodes (visit counts equal the oracle's), the
    warp fetches equal the Fig.8 union, accelerations within 1e-4."""
    b, ot, ref, tree = bh_small
    bd = dev(b)
    order = P.tt_sort_points(tree, bd) if sorted_ else None
    st = P.Stats.alloc(len(b), "cuda")
    acc = P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=order, mode=mode, stats=st, variant="groups").cpu().numpy()
    err = rel_err(acc, ref.out[0])
    assert err.max() <= BH_TOL, err.max()
    assert np.array_equal(st.visits.cpu().numpy(), ref.visits)
    if mode == "lockstep":
        o = order.cpu().numpy() if sorted_ else np.arange(len(b))
        union = oracle.unguided_warp_union(ot, b[o], 0.5, W=32 * P._lib.BH_POINTS_PER_LANE)
        assert np.array_equal(st.warp_fetches.cpu().numpy()[:len(union)], union)


def test_bh_groups_theta0_buckets_and_1m():
    from tests import brute
    b = ttgen.plummer(3001, seed=204)
    b[100, :3] = b[101, :3] = b[102, :3]  # a depth-32 bucket
    tree = P.tt_tree_upload(P.build_oct(b))
    acc = P.tt_traverse_bh(tree, dev(b), 0.0, 0.05, mode="lockstep", variant="groups").cpu().numpy()
    assert rel_err(acc, brute.direct_sum(b, 0.05)).max() <= BH_TOL
    c = ttgen.CONFIGS["bh_1m_plummer"]
    b = ttgen.plummer(c["n"], c["seed"])
    tree = P.tt_build_oct_device(dev(b))
    bd = dev(b)
    perm = P.tt_sort_points(tree, bd)
    acc = P.tt_traverse_bh(tree, bd, c["theta"], c["eps"], order=perm, variant="groups").cpu().numpy()
    sample = np.concatenate([np.random.default_rng(5).choice(len(b), 3000, replace=False),
                             np.argsort(np.linalg.norm(b[:, :3], axis=1))[:500]])
    ref = oracle.bh(oracle.build_oct(b), b[sample], c["theta"], c["eps"], self_ids=sample)
    assert rel_err(acc[sample], ref.out[0]).max() <= BH_TOL


def test_bh_group_arrays_recycled_across_trees():
    """Child-group arrays are returned to a small cache when a tree is freed
    and reused by later trees (time stepping builds one per step): trees of
    changing sizes, each checked against the oracle."""
    import gc
    for n, seed in ((20011, 1), (3, 2), (20011, 3), (50000, 4), (777, 5), (20011, 6)):
        b = ttgen.plummer(n, seed=300 + seed)
        tree = P.tt_build_oct_device(dev(b))
        acc = P.tt_traverse_bh(tree, dev(b), 0.5, 0.05, mode="lockstep").cpu().numpy()
        ref = oracle.bh(oracle.build_oct(b), b, 0.5, 0.05, self_ids=np.arange(n))
        assert rel_err(acc, ref.out[0]).max() <= BH_TOL, n
        tree.free()
        del tree
        gc.collect()


def test_bh_default_falls_back_for_trees_deeper_than_group_stack(bh_small):
    """A custom tree whose declared height exceeds the child-group stack
    (8 entries per level) but not TT_MAX_HEIGHT: the default BH path takes the
    per-node rope walk (same visits, within 1e-4); an explicit request for
    the child-group walk fails with TT_ERR_TREE_TOO_DEEP."""
    b, ot, ref, _ = bh_small
    h = P.build_oct(b)
    h.desc.height = P._lib.MAX_HEIGHT  # legal for the pack, too deep for the group stack
    tree = P.tt_tree_upload(h)
    bd = dev(b)
    st = P.Stats.alloc(len(b), "cuda")
    acc = P.tt_traverse_bh(tree, bd, 0.5, 0.05, mode="lockstep", stats=st).cpu().numpy()
    assert rel_err(acc, ref.out[0]).max() <= BH_TOL
    assert np.array_equal(st.visits.cpu().numpy(), ref.visits)
    with pytest.raises(P.TTError) as e:
        P.tt_traverse_bh(tree, bd, 0.5, 0.05, variant="groups")
    assert e.value.status == -4


@pytest.mark.parametrize("case,variant", [("shifted", "autoropes"), ("eps0", "autoropes"), ("foreign_ids", "autoropes"),
                                          ("eps0", "ropes"), ("eps0_no_self", "autoropes")])
def test_bh_groups_self_test_only_where_it_matters(case, variant):
    """The child-group walk drops its per-child self test in warps whose bodies
    all sit exactly on their own leaves with eps > 0 (that leaf's term is then
    f * 0 = 0).  Warps where that does not hold keep the test: queries moved
    off their leaves (every other warp tile), eps = 0 (the term would be
    inf * 0), and self ids naming other bodies' leaves."""
    b = ttgen.plummer(20011, seed=311)
    ot = oracle.build_oct(b)
    tree = P.tt_tree_upload(P.build_oct(b))
    q = b.copy()
    ids = np.arange(len(b))
    eps = 0.05
    if case == "shifted":
        moved = (np.arange(len(b)) // 64) % 2 == 1
        q[moved, :3] += np.float32(1e-3)
    elif case == "eps0":
        eps = 0.0
    elif case == "eps0_no_self":
        # self ids naming no leaf and eps = 0: queries strictly inside the
        # cloud, off every body (a body's own leaf would be a 1/0 term)
        eps = 0.0
        ids = np.full(len(b), -1)
        q = q[:4096].copy()
        q[:, :3] = (q[:, :3] * np.float32(0.5) + np.float32(1e-4)).astype(np.float32)
        ids = ids[:4096]
    else:
        ids = np.roll(ids, 1)
    acc = P.tt_traverse_bh(tree, dev(q), 0.5, eps, self_ids=perm_i32(ids), mode="lockstep",
                           variant=variant).cpu().numpy()
    ref = oracle.bh(ot, q, 0.5, eps, self_ids=ids)
    assert np.isfinite(acc).all() and np.isfinite(ref.out[0]).all()
    assert rel_err(acc, ref.out[0]).max() <= BH_TOL


@pytest.mark.parametrize("dup", [9, 40])
@pytest.mark.parametrize("builder", ["host", "device"])
def test_bh_groups_wide_buckets(dup, builder):
    """A depth-32 bucket (R9) of more than 8 coincident bodies: its cell has
    `dup` leaf children, more than the 8-record staging buffer of the
    child-group walk, which then stages groups 8 at a time (header
    oct_flags without TT_OCT_NARROW).  Every mode against the oracle: visits
    exact, accelerations within 1e-4 (theta = 0.5 and theta = 0)."""
    b = ttgen.plummer(5003, seed=320 + dup)
    b[200:200 + dup, :3] = b[7, :3]
    b[3000:3000 + dup, :3] = b[4000, :3]  # and a second one in another warp tile
    ot = oracle.build_oct(b)
    assert ot.height == 33
    tree = P.tt_tree_upload(P.build_oct(b)) if builder == "host" else P.tt_build_oct_device(dev(b))
    bd = dev(b)
    for theta in (0.5, 0.0):
        ref = oracle.bh(ot, b, theta, 0.05, self_ids=np.arange(len(b)), stats=True)
        for mode in MODES:
            st = P.Stats.alloc(len(b), "cuda")
            acc = P.tt_traverse_bh(tree, bd, theta, 0.05, mode=mode, stats=st).cpu().numpy()
            assert rel_err(acc, ref.out[0]).max() <= BH_TOL, (theta, mode)
            assert np.array_equal(st.visits.cpu().numpy(), ref.visits), (theta, mode)
        if theta == 0.5:
            st = P.Stats.alloc(len(b), "cuda")
            P.tt_traverse_bh(tree, bd, theta, 0.05, mode="lockstep", stats=st)
            union = oracle.unguided_warp_union(ot, b, 0.5, W=32 * P._lib.BH_POINTS_PER_LANE)
            assert np.array_equal(st.warp_fetches.cpu().numpy()[:len(union)], union)

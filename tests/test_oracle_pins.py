"""Pins of the CPU oracle against things other than itself (runs without a GPU).

Each test names the passage (PAPER.md P:Lx-y) or the mathematical fact it
pins.  These must pass before any CUDA result is compared with the oracle.
"""
from __future__ import annotations

import os

import numpy as np
import pytest

import oracle
import ttgen
from tests import brute

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ---------------------------------------------------------------- Fig.2 ropes
def test_fig2_linearisation_and_ropes():
    """Left-biased linearisation + ropes of the Fig.2 worked example."""
    rows = []
    for line in open(os.path.join(GOLDEN, "fig2_ropes.txt")):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        lhs, rhs = line.split("|")
        lab, *ch = [int(x) for x in lhs.split()]
        pre, skip = [int(x) for x in rhs.split()]
        rows.append((lab, ch, pre, skip))
    labels = [r[0] for r in rows]
    children = [[labels.index(c) for c in r[1]] for r in rows]
    t = oracle.build_generic(children, root=0)
    got_label = t.i64(oracle.F_LABEL)  # label index (0-based) in preorder
    got_skip = t.i64(oracle.F_SKIP)
    for lab, ch, pre, skip in rows:
        p = pre - 1
        assert labels[got_label[p]] == lab
        assert got_skip[p] + 1 == skip
    # guided push order at node 1 is "first 5, then 2": reversed children
    assert [labels[c] for c in reversed(children[0])] == [5, 2]


def _subtree_sizes(ch):
    n = len(ch)
    size = np.ones(n, np.int64)
    for v in range(n - 1, -1, -1):
        for c in ch[v]:
            if c >= 0:
                size[v] += size[c]
    return size


def _check_preorder_skip(t):
    """skip[n] = n + |subtree(n)| and first child = n + 1 (preorder)."""
    ch = t.children()
    size = _subtree_sizes(ch)
    skip = t.i64(oracle.F_SKIP)
    assert np.array_equal(skip, np.arange(t.n_nodes) + size)
    for v in range(t.n_nodes):
        kids = [c for c in ch[v] if c >= 0]
        if kids:
            assert kids[0] == v + 1
            # each next child starts where the previous subtree ends
            for a, b in zip(kids, kids[1:]):
                assert b == skip[a]


# ------------------------------------------------------------------ kd-tree
@pytest.mark.parametrize("n,dim,leaf", [(2000, 3, 1), (3000, 7, 8), (777, 2, 3)])
def test_kd_build_invariants(n, dim, leaf):
    p = ttgen.gaussian_mixture(n, dim, seed=11, components=4)
    p[::50] = p[0]  # duplicates
    t = oracle.build_kd(p, leaf)
    _check_preorder_skip(t)
    order = t.tree_order()
    assert np.array_equal(np.sort(order), np.arange(n))  # every point in exactly one leaf
    pb, pc_ = t.i64(oracle.F_PBEGIN), t.i64(oracle.F_PCOUNT)
    sd, split = t.i64(oracle.F_SPLITDIM), t.f32(oracle.F_SPLIT)
    lo, hi = t.f32(oracle.F_LO, dim), t.f32(oracle.F_HI, dim)
    ch = t.children()
    for v in range(t.n_nodes):
        pts = p[order[pb[v]:pb[v] + pc_[v]]]
        assert np.array_equal(lo[v], pts.min(0)) and np.array_equal(hi[v], pts.max(0))  # tight box
        if sd[v] < 0:
            assert 1 <= pc_[v] <= leaf
            continue
        ext = (hi[v] - lo[v]).astype(np.float32)
        assert sd[v] == int(np.argmax(ext))  # largest extent, lowest dim on ties
        L, R = ch[v, 0], ch[v, 1]
        assert pc_[L] == pc_[v] // 2 and pc_[R] == pc_[v] - pc_[v] // 2  # median split
        lp = p[order[pb[L]:pb[L] + pc_[L]], sd[v]]
        rp = p[order[pb[R]:pb[R] + pc_[R]], sd[v]]
        assert lp.max() <= split[v] <= rp.min()
        assert split[v] in rp


# ------------------------------------------------------------------ oct-tree
def test_oct_build_invariants():
    b = ttgen.plummer(3000, seed=12)
    t = oracle.build_oct(b)
    _check_preorder_skip(t)
    order = t.tree_order()
    assert np.array_equal(np.sort(order), np.arange(len(b)))
    c, side = t.root_cube()
    codes = brute.morton63(b, c, side)
    pb, pcn, lvl = t.i64(oracle.F_PBEGIN), t.i64(oracle.F_PCOUNT), t.i64(oracle.F_LEVEL)
    body = t.i64(oracle.F_BODY)
    com = np.stack([t.f32(oracle.F_COMX), t.f32(oracle.F_COMY), t.f32(oracle.F_COMZ)], 1)
    mass = t.f32(oracle.F_MASS)
    ch = t.children()
    for v in range(t.n_nodes):
        ids = order[pb[v]:pb[v] + pcn[v]]
        # all bodies of a node share the octant path of its depth (cube containment)
        sh = np.uint64(63 - 3 * lvl[v])
        if lvl[v] > 0:
            assert len(np.unique(codes[ids] >> sh)) == 1
        kids = [k for k in ch[v] if k >= 0]
        if body[v] >= 0:
            assert pcn[v] == 1 and ids[0] == body[v] and not kids
        else:
            assert len(kids) >= 1  # a cell may hold a single non-empty octant
            # children in increasing octant order
            octs = [int((codes[order[pb[k]]] >> np.uint64(63 - 3 * (lvl[v] + 1))) & np.uint64(7)) for k in kids]
            assert octs == sorted(octs) and len(set(octs)) == len(octs)
        # COM = mass-weighted mean of the bodies (fp64 brute), rounded to fp32
        bb = b[ids].astype(np.float64)
        M = bb[:, 3].sum()
        want = (bb[:, :3] * bb[:, 3:4]).sum(0) / M
        np.testing.assert_allclose(com[v], want, rtol=2e-6, atol=1e-6)
        np.testing.assert_allclose(mass[v], M, rtol=2e-7)


def test_oct_bucket_for_identical_bodies():
    """Identical positions cannot be separated: a bucket cell at depth 32 (R9)."""
    b = ttgen.plummer(64, seed=13)
    b[5, :3] = b[6, :3] = b[7, :3]
    t = oracle.build_oct(b)
    assert t.height == 33
    assert np.array_equal(np.sort(t.tree_order()), np.arange(64))


# ------------------------------------------------------------------- vp-tree
def test_vp_build_invariants():
    p = ttgen.gaussian_mixture(1500, 5, seed=14, components=3)
    t = oracle.build_vp(p)
    _check_preorder_skip(t)
    order = t.tree_order()
    assert np.array_equal(np.sort(order), np.arange(len(p)))
    vp, rin, rout = t.i64(oracle.F_VP), t.f32(oracle.F_RIN), t.f32(oracle.F_ROUT)
    pb, pcn = t.i64(oracle.F_PBEGIN), t.i64(oracle.F_PCOUNT)
    ch = t.children()
    for v in range(t.n_nodes):
        ids = order[pb[v]:pb[v] + pcn[v]]
        assert ids[0] == vp[v] == ids.min()  # vantage = smallest id of the set
        d = np.sqrt(brute.pinned_d2(p[[vp[v]]], p)[0])
        cin, cout = ch[v, 0], ch[v, 1]
        nrest = pcn[v] - 1
        if cin >= 0:
            ii = order[pb[cin]:pb[cin] + pcn[cin]]
            assert len(ii) == nrest // 2
            assert np.all(d[ii] <= rin[v]) and rin[v] in d[ii]
        if cout >= 0:
            oo = order[pb[cout]:pb[cout] + pcn[cout]]
            assert np.all(d[oo] >= rout[v]) and rout[v] in d[oo]
        if cin >= 0 and cout >= 0:
            assert rin[v] <= rout[v]


# ------------------------------------------------------------------------ PC
def test_pc_vs_bruteforce():
    """Fig.4 recursion == all-pairs count (R1 closed ball, self counted)."""
    p = ttgen.uniform(2048, 3, seed=21)
    p[100:110] = p[5]  # exact duplicates sit on the boundary of every test
    t = oracle.build_kd(p, 1)
    for r in (0.0, 0.05, 0.1, 0.3):
        got = oracle.pc(t, p, r).out[0]
        assert np.array_equal(got, brute.pc_counts(p, p, r))
        assert got.min() >= 1
        # the pair relation is symmetric: rn(a-b) = -rn(b-a), so the number of
        # ordered pairs i != j is even
        assert (int(got.sum()) - len(p)) % 2 == 0


def test_pc_bucket_leaves_and_queries():
    p = ttgen.gaussian_mixture(3000, 7, seed=22, components=5)
    q = ttgen.gaussian_mixture(500, 7, seed=23, components=5)
    t = oracle.build_kd(p, 8)
    got = oracle.pc(t, q, 0.12).out[0]
    assert np.array_equal(got, brute.pc_counts(q, p, 0.12))
    assert np.array_equal(oracle.pc(t, q, np.inf).out[0], np.full(len(q), len(p)))  # r = inf -> N
    # monotone in r
    a = oracle.pc(t, q, 0.05).out[0]
    assert np.all(a <= got)


def test_pc_visit_count_matches_paper_shape():
    """Config 1 shape: ~220 visits/point, count ~38 (sanity, not parity)."""
    p = ttgen.uniform(10_000, 3, seed=1)
    t = oracle.build_kd(p, 1)
    r = oracle.pc(t, p, 0.1, stats=True)
    assert 150 < r.visits.mean() < 300
    assert 30 < r.out[0].mean() < 45
    assert t.n_nodes == 19_999


# ------------------------------------------------------------------------ BH
def test_bh_theta0_equals_direct_sum():
    """theta = 0 -> dsq = +inf -> every cell opened -> O(n^2) direct sum (R8)."""
    b = ttgen.plummer(1500, seed=31)
    t = oracle.build_oct(b)
    assert oracle.bh_dsq_root(t, 0.0) == np.inf
    got = oracle.bh(t, b, 0.0, 0.05, self_ids=np.arange(len(b))).out[0]
    want = brute.direct_sum(b, 0.05)
    err = np.linalg.norm(got - want, axis=1) / np.linalg.norm(want, axis=1)
    assert err.max() < 1e-11


def test_bh_two_body_closed_form():
    """a_0 = m_1 r / (r^2 + eps^2)^{3/2} for two bodies whenever the root cell
    opens (theta <= 0.5 here; at larger theta the root is 'far enough' and each body
    sees the root monopole, which includes itself -- Fig.9a has no self test
    for cells)."""
    b = np.array([[0.1, 0.2, 0.3, 0.5], [0.4, -0.2, 0.7, 0.25]], np.float32)
    t = oracle.build_oct(b)
    for theta in (0.0, 0.25, 0.5):
        a = oracle.bh(t, b, theta, 0.05, self_ids=np.arange(2)).out[0]
        x = b.astype(np.float64)
        r = x[1, :3] - x[0, :3]
        e2 = float(np.float32(0.05)) ** 2
        np.testing.assert_allclose(a[0], x[1, 3] * r / (r @ r + e2) ** 1.5, rtol=1e-14)
        np.testing.assert_allclose(a[1], -x[0, 3] * r / (r @ r + e2) ** 1.5, rtol=1e-14)


def test_bh_theta0_momentum_and_duplicates():
    """Newton's third law: sum_i m_i a_i = 0 at theta = 0, incl. a depth-32 bucket."""
    b = ttgen.plummer(600, seed=32)
    b[10, :3] = b[11, :3] = b[12, :3]
    t = oracle.build_oct(b)
    a = oracle.bh(t, b, 0.0, 0.05, self_ids=np.arange(len(b))).out[0]
    mom = (b[:, 3:4].astype(np.float64) * a).sum(0)
    assert np.abs(mom).max() < 1e-12 * np.abs(b[:, 3:4] * a).sum()
    want = brute.direct_sum(b, 0.05)
    err = np.linalg.norm(a - want, axis=1) / np.linalg.norm(want, axis=1)
    assert err.max() < 1e-11


def test_bh_theta_half_approximation_is_small():
    """theta = 0.5 monopole BH vs direct sum: characterises the approximation
    (not parity): median error well below 1e-2."""
    b = ttgen.plummer(4000, seed=33)
    t = oracle.build_oct(b)
    a = oracle.bh(t, b, 0.5, 0.05, self_ids=np.arange(len(b))).out[0]
    want = brute.direct_sum(b, 0.05)
    err = np.linalg.norm(a - want, axis=1) / np.linalg.norm(want, axis=1)
    assert np.median(err) < 1e-2


# ----------------------------------------------------------------------- kNN
@pytest.mark.parametrize("k", [1, 8, 17])
def test_knn_vs_bruteforce(k):
    p = ttgen.gaussian_mixture(2048, 7, seed=41, components=6)
    p[200:205] = p[3]  # ties broken by index (R4)
    q = np.concatenate([ttgen.gaussian_mixture(400, 7, seed=42, components=6), p[:100]])
    t = oracle.build_kd(p, 8)
    idx, d2 = oracle.knn(t, q, k).out
    bidx, bd2 = brute.knn(q, p, k)
    assert np.array_equal(idx, bidx)
    assert np.array_equal(d2, bd2)
    assert np.all(np.diff(d2, axis=1) >= 0)  # sorted ascending
    # pinned fp32 d2 is within D*u relative of the exact distance
    exact = ((q[:, None, :].astype(np.float64) - p[idx].astype(np.float64)) ** 2).sum(-1)
    assert np.all(np.abs(d2 - exact) <= 7 * 2.0 ** -23 * exact + 1e-30)


def test_knn_k_exceeds_n_pads():
    p = ttgen.uniform(5, 3, seed=43)
    t = oracle.build_kd(p, 2)
    idx, d2 = oracle.knn(t, p, 8).out
    assert np.all(idx[:, 5:] == -1) and np.all(np.isinf(d2[:, 5:]))
    assert np.array_equal(np.sort(idx[:, :5], 1), np.tile(np.arange(5), (5, 1)))


def test_knn_cross_kernel_with_pc():
    """With r2 := d2_k(q): PC count >= k; with the next float below: count < k."""
    p = ttgen.gaussian_mixture(1500, 3, seed=44, components=4)
    t1 = oracle.build_kd(p, 1)
    t8 = oracle.build_kd(p, 8)
    k = 8
    idx, d2 = oracle.knn(t8, p[:200], k).out
    for i in range(200):
        rk = float(np.sqrt(np.float64(d2[i, -1])))
        # radius whose fp32 square is >= d2_k ...
        r = np.float32(rk)
        while np.float32(r * r) < d2[i, -1]:
            r = np.nextafter(r, np.float32(np.inf))
        assert oracle.pc(t1, p[i:i + 1], float(r)).out[0][0] >= k
        r = np.float32(rk)
        while np.float32(r * r) >= d2[i, -1]:
            r = np.nextafter(r, np.float32(0))
        assert oracle.pc(t1, p[i:i + 1], float(r)).out[0][0] < k


# ------------------------------------------------------------------------ VP
def test_vp_vs_bruteforce_and_knn1():
    p = ttgen.gaussian_mixture(2000, 16, seed=51, components=8)
    p[300:303] = p[7]
    q = np.concatenate([ttgen.gaussian_mixture(300, 16, seed=52, components=8), p[:50]])
    t = oracle.build_vp(p)
    idx, d2 = oracle.vp(t, q).out
    bidx, bd2 = brute.nn(q, p)
    assert np.array_equal(idx, bidx) and np.array_equal(d2, bd2)
    kt = oracle.build_kd(p, 8)
    kidx, kd2 = oracle.knn(kt, q, 1).out
    assert np.array_equal(kidx[:, 0], idx) and np.array_equal(kd2[:, 0], d2)


# ---------------------------------------------------------------- autoropes
def test_visits_each_node_at_most_once_and_order_hash_stable():
    """Each node tested at most once per traversal: visits <= n_nodes;
    N-mode counts do not depend on the order points are processed (Table 1:
    N rows identical sorted vs unsorted, e.g. P:L1154, L1166, L1178, L1202)."""
    p = ttgen.uniform(3000, 3, seed=61)
    t = oracle.build_kd(p, 1)
    r = oracle.pc(t, p, 0.15, stats=True)
    assert r.visits.max() <= t.n_nodes
    perm = ttgen.permutation(len(p), 62)
    r2 = oracle.pc(t, p[perm], 0.15, stats=True)
    assert np.array_equal(r2.visits, r.visits[perm]) and np.array_equal(r2.hash, r.hash[perm])


# --------------------------------------------------------------------- sort
def test_sort_keys_kd_reproduce_tree_order():
    p = ttgen.uniform(4096, 3, seed=71)
    t = oracle.build_kd(p, 1)
    perm = oracle.sort_perm(t, p)
    assert np.array_equal(perm, t.tree_order())  # descent of a data point ends at its own leaf


def test_sort_keys_oct_follow_the_hilbert_curve():
    """Oct sort keys (reading R18b) order the points' 16-level cells of the
    cube hierarchy along a Hilbert curve.  Pinned by the curve's defining
    properties, not by its formula: (1) consecutive cells are face-adjacent
    -- a grid of 8^3 bodies, one per level-3 cell of the unit root cube,
    sorted by key steps by exactly one cell along one axis each time; (2)
    the curve fills every dyadic cube before leaving it -- for Plummer bodies
    each level-k cell (Morton prefix, the build's octant rule) is one
    contiguous run of the sorted order, k = 1..7; (3) one key per cell."""
    g = (np.stack(np.meshgrid(np.arange(8), np.arange(8), np.arange(8), indexing="ij"), -1).reshape(-1, 3) + 0.5) / 8
    corners = np.array([[0, 0, 0], [1, 1, 1]], np.float64)  # make the root cube exactly [0, 1]^3
    pts = np.concatenate([g, corners])
    b = np.concatenate([pts, np.ones((len(pts), 1))], 1).astype(np.float32)
    t = oracle.build_oct(b)
    c, side = t.root_cube()
    assert side == 1.0 and np.array_equal(c, [0.5, 0.5, 0.5])
    keys = oracle.sort_keys(t, b)[:512]
    o = np.argsort(keys, kind="stable")
    cells = np.floor(g[o] * 8).astype(int)
    assert np.all(np.abs(np.diff(cells, axis=0)).sum(1) == 1)
    assert len(np.unique(keys)) == 512

    bp = ttgen.plummer(5000, seed=72)
    t = oracle.build_oct(bp)
    c, side = t.root_cube()
    hk = oracle.sort_keys(t, bp)
    mk = brute.morton63(bp, c, side)
    o = np.argsort(hk, kind="stable")
    for k in range(1, 8):
        pre = (mk[o] >> np.uint64(63 - 3 * k))
        starts = np.concatenate([[True], pre[1:] != pre[:-1]])
        assert starts.sum() == len(np.unique(pre)), k  # each level-k cell is one run
    lv16 = mk >> np.uint64(63 - 48)
    assert len(np.unique(hk)) == len(np.unique(lv16))  # one key per 16-level cell
    assert hk.max() < 2 ** 48


def test_sort_keys_vp_are_a_stable_bijection():
    p = ttgen.gaussian_mixture(3000, 16, seed=73, components=4)
    t = oracle.build_vp(p)
    keys = oracle.sort_keys(t, p)
    perm = oracle.sort_perm(t, p)
    assert np.array_equal(np.sort(perm), np.arange(len(p)))
    ks = keys[perm]
    assert np.all(ks[1:] >= ks[:-1])
    # equal keys keep input order (stability)
    same = ks[1:] == ks[:-1]
    assert np.all(perm[1:][same] > perm[:-1][same])


# ----------------------------------------------------------------- lockstep
def test_unguided_lockstep_union_and_work_expansion():
    """Work expansion = warp fetches / longest lane traversal >= 1;
    sorting lowers it (Table 2)."""
    b = ttgen.plummer(8192, seed=81)
    t = oracle.build_oct(b)
    r = oracle.bh(t, b, 0.5, 0.05, self_ids=np.arange(len(b)), stats=True)
    perm = oracle.sort_perm(t, b)
    for order in (perm, ttgen.permutation(len(b), 82)):
        wf = oracle.unguided_warp_union(t, b[order], 0.5)
        lv = r.visits[order].reshape(-1, 32)
        assert np.all(wf >= lv.max(1)) and np.all(wf <= lv.sum(1))
    ws = (oracle.unguided_warp_union(t, b[perm], 0.5) / r.visits[perm].reshape(-1, 32).max(1)).mean()
    wu = (oracle.unguided_warp_union(t, b[ttgen.permutation(len(b), 82)], 0.5)
          / r.visits[ttgen.permutation(len(b), 82)].reshape(-1, 32).max(1)).mean()
    assert 1.0 <= ws < wu


def test_guided_lockstep_results_equal_independent():
    """Majority-vote call-set reduction does not change results."""
    p = ttgen.gaussian_mixture(3000, 7, seed=91, components=6)
    q = ttgen.gaussian_mixture(1000, 7, seed=92, components=6)
    kt = oracle.build_kd(p, 8)
    for qq in (q, q[oracle.sort_perm(kt, q)]):
        idx, d2 = oracle.knn(kt, qq, 8).out
        li, ld, lv, wf = oracle.knn_lockstep(kt, qq, 8)
        assert np.array_equal(li, idx) and np.array_equal(ld, d2)
        assert np.all(wf >= 1)
    p16 = ttgen.gaussian_mixture(2000, 16, seed=93, components=6)
    q16 = ttgen.gaussian_mixture(700, 16, seed=94, components=6)
    vt = oracle.build_vp(p16)
    idx, d2 = oracle.vp(vt, q16).out
    li, ld, lv, wf = oracle.vp_lockstep(vt, q16)
    assert np.array_equal(li, idx) and np.array_equal(ld, d2)


# ------------------------------------------------ NN kd-tree (NEXT-3, R21)
@pytest.mark.parametrize("n,dim", [(1500, 3), (2001, 7), (64, 16), (1, 4), (2, 2)])
def test_nn_build_invariants(n, dim):
    """Point-per-node kd-tree (the paper's NN; build rule R21):
    preorder/ropes, every point at exactly one node, the node's point is the
    median of its set on (x[dim], id) along the largest-extent dimension."""
    p = ttgen.gaussian_mixture(n, dim, seed=15, components=3)
    if n > 100:
        p[50:60] = p[3]  # exact duplicates: ties on x[dim] broken by id
    t = oracle.build_nn(p)
    _check_preorder_skip(t)
    order = t.tree_order()
    assert np.array_equal(np.sort(order), np.arange(n))
    assert t.n_nodes == n
    pb, pcn = t.i64(oracle.F_PBEGIN), t.i64(oracle.F_PCOUNT)
    sd, split, me = t.i64(oracle.F_SPLITDIM), t.f32(oracle.F_SPLIT), t.i64(oracle.F_VP)
    lo, hi = t.f32(oracle.F_LO, dim).reshape(-1, dim), t.f32(oracle.F_HI, dim).reshape(-1, dim)
    ch = t.children()
    for v in range(t.n_nodes):
        ids = order[pb[v]:pb[v] + pcn[v]]
        assert ids[0] == me[v]  # the node's own point first, then its subtrees
        assert np.array_equal(lo[v], p[ids].min(0)) and np.array_equal(hi[v], p[ids].max(0))  # tight box
        if len(ids) == 1:
            assert sd[v] == -1 and ch[v, 0] == -1 and ch[v, 1] == -1
            continue
        ext = (p[ids].max(0) - p[ids].min(0)).astype(np.float32)
        assert sd[v] == int(np.argmax(ext))  # largest extent, lowest dim on ties
        d = sd[v]
        srt = sorted(ids, key=lambda i: (p[i, d], i))
        m = len(ids) // 2
        assert srt[m] == me[v] and split[v] == p[me[v], d]
        left = order[pb[ch[v, 0]]:pb[ch[v, 0]] + pcn[ch[v, 0]]] if ch[v, 0] >= 0 else []
        right = order[pb[ch[v, 1]]:pb[ch[v, 1]] + pcn[ch[v, 1]]] if ch[v, 1] >= 0 else []
        assert sorted(left) == sorted(srt[:m]) and sorted(right) == sorted(srt[m + 1:])
        assert all(p[i, d] <= split[v] for i in left) and all(p[i, d] >= split[v] for i in right)


def test_nn_vs_bruteforce_knn1_and_vp():
    """NN = argmin (d2, id) (the plain definition); the same
    answer as kNN with k = 1 and as the vantage-point tree (three different
    trees and pruning rules)."""
    for dim, seed in ((7, 53), (16, 54), (3, 55)):
        p = ttgen.gaussian_mixture(2500, dim, seed=seed, components=8)
        p[400:404] = p[9]
        q = np.concatenate([ttgen.gaussian_mixture(400, dim, seed=seed + 100, components=8), p[:60]])
        t = oracle.build_nn(p)
        r = oracle.nn(t, q, stats=True)
        idx, d2 = r.out
        bidx, bd2 = brute.nn(q, p)
        assert np.array_equal(idx, bidx) and np.array_equal(d2, bd2)
        kidx, kd2 = oracle.knn(oracle.build_kd(p, 8), q, 1).out
        assert np.array_equal(kidx[:, 0], idx) and np.array_equal(kd2[:, 0], d2)
        vidx, vd2 = oracle.vp(oracle.build_vp(p), q).out
        assert np.array_equal(vidx, idx) and np.array_equal(vd2, d2)
        assert r.visits.max() <= t.n_nodes and r.visits.min() >= 1
        if dim <= 7:  # the box bound prunes: far fewer tests than nodes
            assert r.visits.mean() < 0.2 * t.n_nodes


def test_nn_visits_order_invariant_and_lockstep_results():
    """N-mode visit counts and the order hash do not depend on the point order
    (P:L1154-1202 N rows); lockstep with majority vote gives the same results
    (P:L847-849)."""
    p = ttgen.gaussian_mixture(3000, 7, seed=56, components=6)
    q = ttgen.gaussian_mixture(900, 7, seed=57, components=6)
    t = oracle.build_nn(p)
    r = oracle.nn(t, q, stats=True)
    perm = ttgen.permutation(len(q), 58)
    r2 = oracle.nn(t, q[perm], stats=True)
    assert np.array_equal(r2.visits, r.visits[perm]) and np.array_equal(r2.hash, r.hash[perm])
    keys = oracle.sort_keys(t, q)
    sp = oracle.sort_perm(t, q)
    assert np.array_equal(np.sort(sp), np.arange(len(q))) and np.all(np.diff(keys[sp].astype(np.float64)) >= 0)
    for qq in (q, q[sp]):
        idx, d2 = oracle.nn(t, qq).out
        li, ld, lv, wf = oracle.nn_lockstep(t, qq)
        assert np.array_equal(li, idx) and np.array_equal(ld, d2)
        assert np.all(wf >= 1) and np.all(wf <= lv.reshape(-1) .sum() + 1)
    # sorting makes lockstep warps cheaper (Table 2)
    wf_s = oracle.nn_lockstep(t, q[sp])[3].mean()
    wf_u = oracle.nn_lockstep(t, q)[3].mean()
    assert wf_s < wf_u


# ------------------------------------------- BH opening test (R8) pinned by hand
# Four unit-mass bodies; bbox [0,1]^3, so the root cube has side 1 and centre
# (0.5, 0.5, 0.5) (R8a).  Octant rule (x>=cx)|(y>=cy)<<1|(z>=cz)<<2:
#   root (L0) -> X (octant 0, L1: A, C) and Y (octant 7, L1: B1, B2)
#   X: centre 0.25, side 0.5: A=(0,0,0) octant 0, C=(0.25,0,0) octant 1 -> two leaves (L2)
#   Y: B1=(1,1,1), B2=(0.95,1,1) share octant 7 at centres 0.75, 0.875, 0.9375 and
#      separate at 0.96875 (B2 octant 6, B1 octant 7): Y (L1) -> Y2 (L2) -> Y3 (L3)
#      -> Y4 (L4) -> leaves B2, B1 (L5)
# Preorder: root 0, X 1, A 2, C 3, Y 4, Y2 5, Y3 6, Y4 7, B2 8, B1 9.
# COM(X) = (0.125, 0, 0), COM(Y..Y4) = (0.975, 1, 1), mass 2 each.
# theta = 0.5: dsq_root = (1/0.5)^2 = 4, dsq_L = 4 * 0.25^L = 1, 0.25, 0.0625, ...
# (Fig.9a/b: dsq*0.25 per level; distance to the COM, node0 =
# "position vector ... and its type"; open iff drsq < dsq_L).
_R8_BODIES = np.array([[0, 0, 0, 1], [0.25, 0, 0, 1], [1, 1, 1, 1], [0.95, 1, 1, 1]], np.float32)
_R8_COM = {1: (np.array([0.125, 0, 0], np.float32), 2.0), 4: (np.array([0.975, 1, 1], np.float32), 2.0)}
for _v in (5, 6, 7):
    _R8_COM[_v] = _R8_COM[4]
# query -> (tested preorder sequence, interacting nodes) under reading R8
_R8_CASES = [
    # |q - COM(X)|^2 = 1.5 >= dsq_1 = 1: X not opened (a 0.5-per-level factor, dsq_1 = 2, would open it)
    ((0.125 - np.sqrt(1.5), 0.0, 0.0), [0, 1, 4], [1, 4]),
    # |q - COM(X)|^2 = 1 exactly: strict "<" keeps X closed ("<=" would open it)
    ((1.125, 0.0, 0.0), [0, 1, 4], [1, 4]),
    # |q - COM(Y)|^2 = 0.45^2 = 0.2025: opens Y (< 1) and Y2 (< 0.25), not Y3 (>= 0.0625)
    # (0.5 per level would also open Y3 and Y4: 8 tests)
    ((0.975, 1.0, 0.55), [0, 1, 4, 5, 6], [1, 6]),
    # 1.05 from COM(X) towards X's cube centre (0.25, 0.25, 0.25): COM distance^2 1.1025
    # keeps X closed, the centre distance^2 0.456 would open it; Y opens (0.43 < 1), Y2 does not
    ((0.125 + 0.35, 0.7, 0.7), [0, 1, 4, 5], [1, 5]),
]


def test_bh_opening_test_hand_worked_example():
    t = oracle.build_oct(_R8_BODIES)
    assert t.n_nodes == 10 and t.height == 5
    c, side = t.root_cube()
    assert side == 1.0 and np.array_equal(c, [0.5, 0.5, 0.5])
    assert oracle.bh_dsq_root(t, 0.5) == 4.0
    assert list(t.i64(oracle.F_LEVEL)) == [0, 1, 2, 2, 1, 2, 3, 4, 5, 5]
    assert list(t.i64(oracle.F_BODY)) == [-1, -1, 0, 1, -1, -1, -1, -1, 3, 2]
    com = np.stack([t.f32(oracle.F_COMX), t.f32(oracle.F_COMY), t.f32(oracle.F_COMZ)], 1)
    for v, (cv, m) in _R8_COM.items():
        assert np.array_equal(com[v], cv) and t.f32(oracle.F_MASS)[v] == m
    eps = 0.05
    e2 = float(np.float32(eps)) ** 2
    for q, seq, inter in _R8_CASES:
        qq = np.array([[*q, 1.0]], np.float32)
        r = oracle.bh(t, qq, 0.5, eps, self_ids=np.array([-1]), stats=True)
        assert r.visits[0] == len(seq), (q, r.visits[0])
        h = 0
        for v in seq:
            h = (h * 31 + v + 1) % 2 ** 64
        assert int(r.hash[0]) == h, q
        want = np.zeros(3)
        x = qq[0, :3].astype(np.float64)
        for v in inter:
            d = _R8_COM[v][0].astype(np.float64) - x
            want += _R8_COM[v][1] * d / (d @ d + e2) ** 1.5
        np.testing.assert_allclose(r.out[0][0], want, rtol=1e-14, atol=0)


def test_bh_error_decreases_with_theta():
    """Monopole BH error vs the O(n^2) direct sum shrinks as the opening angle
    shrinks (theta -> 0 is the direct sum, R8): medians strictly decrease over
    theta = 0.8, 0.5, 0.25, and theta = 0.25 is below 1e-3."""
    from tests import brute
    b = ttgen.plummer(3000, seed=34)
    t = oracle.build_oct(b)
    want = brute.direct_sum(b, 0.05)
    med = []
    for theta in (0.8, 0.5, 0.25):
        a = oracle.bh(t, b, theta, 0.05, self_ids=np.arange(len(b))).out[0]
        med.append(np.median(np.linalg.norm(a - want, axis=1) / np.linalg.norm(want, axis=1)))
    assert med[0] > med[1] > med[2] and med[2] < 1e-3, med


@pytest.fixture(scope="module")
def bh_1m():
    c = ttgen.CONFIGS["bh_1m_plummer"]
    b = ttgen.plummer(c["n"], c["seed"])
    return c, b, oracle.build_oct(b)


def test_bh_1m_visits_per_body_paper_shape(bh_1m):
    """Paper-shape sanity: N-mode nodes per body on the 1M-body
    Plummer sphere at theta = 0.5 within 10% of Table 1's 2,551.
    The paper's generator and tree details differ, so this is a sanity bound
    on the opening test (a per-level factor of 0.5 instead of 0.25, or "<="
    at every level, moves it far outside), not parity."""
    c, b, t = bh_1m
    s = np.arange(0, len(b), 64)
    r = oracle.bh(t, b[s], c["theta"], c["eps"], self_ids=s, stats=True)
    assert abs(r.visits.mean() / 2551 - 1) < 0.10, r.visits.mean()


def test_bh_1m_work_expansion_paper_shape(bh_1m):
    """Table 2 (metric P:L2307-2313): lockstep work expansion of
    32-body warps on Plummer, sorted 1.33 and unsorted 8.97 -- ours within 10%
    (1,000 sorted warps, 200 unsorted ones, sampled)."""
    c, b, t = bh_1m
    perm = oracle.sort_perm(t, b)
    W = 32
    rng = np.random.default_rng(7)
    ws = rng.choice(len(b) // W, 1000, replace=False)
    ids = np.concatenate([perm[w * W:(w + 1) * W] for w in ws])
    up = ttgen.permutation(len(b), 99)[:200 * W]
    we = []
    for sel in (ids, up):
        u = oracle.unguided_warp_union(t, b[sel], c["theta"], W=W)
        v = oracle.bh(t, b[sel], c["theta"], c["eps"], self_ids=sel, stats=True).visits
        e = oracle.work_expansion(u, v, W)
        assert np.all(e >= 1.0)  # the union contains the longest lane's walk
        we.append(e.mean())
    assert abs(we[0] / 1.33 - 1) < 0.10 and abs(we[1] / 8.97 - 1) < 0.10, we


# ------------------------------------------------------ order-insensitive hash
def test_set_hash_is_the_visited_set():
    """set_hash = sum of mix64(pre + 1) over the tested nodes: a walk that
    never truncates (PC with r = inf) tests every node, so its set hash is
    that sum over all nodes; the order hash of that walk is the preorder
    sequence (autoropes keep the recursive order)."""
    p = ttgen.uniform(300, 3, seed=63)
    t = oracle.build_kd(p, 1)
    r = oracle.pc(t, p[:5], np.inf, stats=True)
    M = 2 ** 64

    def mix64(z):
        z ^= z >> 30
        z = (z * 0xbf58476d1ce4e5b9) % M
        z ^= z >> 27
        z = (z * 0x94d049bb133111eb) % M
        return z ^ (z >> 31)
    want_set = sum(mix64(v + 1) for v in range(t.n_nodes)) % M
    want_ord = 0
    for v in range(t.n_nodes):
        want_ord = (want_ord * 31 + v + 1) % M
    assert np.all(r.visits == t.n_nodes)
    assert all(int(x) == want_set for x in r.set_hash)
    assert all(int(x) == want_ord for x in r.hash)
    # and the set hash does not see the order: the same nodes in any order
    perm = ttgen.permutation(len(p), 64)
    r2 = oracle.pc(t, p[perm], 0.2, stats=True)
    r1 = oracle.pc(t, p, 0.2, stats=True)
    assert np.array_equal(r2.set_hash, r1.set_hash[perm])


# ---------------------------------------------- guided lockstep work expansion
@pytest.mark.parametrize("kind", ["knn", "vp", "nn"])
def test_guided_lockstep_work_expansion_at_least_one(kind):
    """Table 2's metric for the guided simulations: nodes the
    lockstep warp tests / nodes of the warp's longest independent traversal.
    Per warp, the warp tests every node any of its lanes tests (>= the longest
    lockstep lane); averaged over warps it is >= 1, sorted and unsorted, and
    sorting lowers it (Table 2).  Nodes expanded (pops with an
    active lane, reading R22) never exceed nodes tested."""
    d = {"knn": 7, "vp": 16, "nn": 7}[kind]
    p = ttgen.gaussian_mixture(4000, d, seed=95, components=6)
    q = ttgen.gaussian_mixture(2048, d, seed=96, components=6)
    t = {"knn": lambda: oracle.build_kd(p, 8), "vp": lambda: oracle.build_vp(p), "nn": lambda: oracle.build_nn(p)}[kind]()
    sp = oracle.sort_perm(t, q)
    we = []
    for qq in (q[sp], q):
        if kind == "knn":
            ind = oracle.knn(t, qq, 8, stats=True)
            ls = oracle.knn_lockstep(t, qq, 8)
        else:
            ind = getattr(oracle, kind)(t, qq, stats=True)
            ls = getattr(oracle, kind + "_lockstep")(t, qq)
        assert np.all(ls.warp_tests >= ls.lane_visits.reshape(-1, 32).max(1))
        assert np.all(ls.warp_fetches <= ls.warp_tests)
        e = oracle.work_expansion(ls.warp_tests, ind.visits)
        we.append(e.mean())
        assert e.mean() >= 1.0
    assert we[0] < we[1], we


@pytest.mark.parametrize("kind", ["knn", "vp", "nn"])
def test_guided_lockstep_lane_hash_equals_independent_when_alone(kind):
    """A lockstep warp of one active lane takes that lane's own near-first
    order at every vote (majority of one), so its lane visits and
    order hash equal the independent (recursive) walk's."""
    d = {"knn": 7, "vp": 16, "nn": 7}[kind]
    p = ttgen.gaussian_mixture(3000, d, seed=97, components=6)
    q = ttgen.gaussian_mixture(31 * 3 + 1, d, seed=98, components=6)[-1:]  # one query, one lane
    t = {"knn": lambda: oracle.build_kd(p, 8), "vp": lambda: oracle.build_vp(p), "nn": lambda: oracle.build_nn(p)}[kind]()
    if kind == "knn":
        ind, ls = oracle.knn(t, q, 8, stats=True), oracle.knn_lockstep(t, q, 8)
    else:
        ind, ls = getattr(oracle, kind)(t, q, stats=True), getattr(oracle, kind + "_lockstep")(t, q)
    assert ls.lane_visits[0] == ind.visits[0] and ls.lane_hash[0] == ind.hash[0]
    assert ls.warp_tests[0] == ind.visits[0]


@pytest.mark.parametrize("dup", [9, 40])
def test_bh_large_bucket_theta0_direct_sum(dup):
    """A depth-32 bucket (R9) holds any number of coincident bodies, one leaf
    child each: at theta = 0 the walk still equals the O(n^2) direct sum."""
    from tests import brute
    b = ttgen.plummer(1200, seed=35 + dup)
    b[100:100 + dup, :3] = b[3, :3]
    t = oracle.build_oct(b)
    assert t.height == 33
    assert np.array_equal(np.sort(t.tree_order()), np.arange(len(b)))
    a = oracle.bh(t, b, 0.0, 0.05, self_ids=np.arange(len(b))).out[0]
    want = brute.direct_sum(b, 0.05)
    assert (np.linalg.norm(a - want, axis=1) / np.linalg.norm(want, axis=1)).max() < 1e-11


# ------------------------------------------------------ VP / NN sort keys (a1)
def _decode_path(key, children):
    """Nodes on the 2-bit-per-level descent code (01 = first child, 10 =
    second, 00 = end; R18), starting at the root."""
    path, v = [0], 0
    for lvl in range(31):
        c = (int(key) >> (62 - 2 * lvl)) & 3
        if c == 0:
            break
        v = int(children[v, c - 1])
        assert v >= 0
        path.append(v)
    return path


def _ancestors(children, n):
    par = np.full(n, -1, np.int64)
    for v in range(n):
        for c in children[v]:
            if c >= 0:
                par[c] = v
    return par


@pytest.mark.parametrize("kind", ["vp", "nn"])
def test_sort_keys_vp_nn_descend_to_the_points_own_node(kind):
    """Pins the VP / NN key paths (R18) against the builders' partitions
    (pinned above by brute force): a data point's descent by the build's
    rule -- VP: inside iff sqrt_rn(d2(vp, x)) <= r_in_max; NN: left iff
    x[dim] < split -- passes through the node holding the point itself, the
    node where it is the vantage / node point.  The only exceptions are the
    boundary ties the rule cannot separate (VP: an outside point at exactly
    r_in_max; NN: a left point with x[dim] == split), each checked to be one.
    Keys sort in preorder of the path's end node (end 00 < 01 < 10)."""
    d = 16 if kind == "vp" else 7
    p = ttgen.gaussian_mixture(3000, d, seed=74, components=5)
    p[40:44] = p[2]  # exact duplicates make boundary ties
    t = oracle.build_vp(p) if kind == "vp" else oracle.build_nn(p)
    keys = oracle.sort_keys(t, p)
    ch = t.children()[:, :2]
    own = np.full(len(p), -1, np.int64)
    own[t.i64(oracle.F_VP)] = np.arange(t.n_nodes)
    par = _ancestors(ch, t.n_nodes)
    pre_end = np.empty(len(p), np.int64)
    exceptions = 0
    for x in range(len(p)):
        path = _decode_path(keys[x], ch)
        pre_end[x] = path[-1]
        if own[x] in path:
            continue
        # walk up from the point's own node: find the ancestor where the rule
        # sends x the other way, and check it is a boundary tie
        v, tie = own[x], False
        while par[v] >= 0:
            a, side = par[v], int(np.where(ch[par[v]] == v)[0][0])
            if kind == "vp":
                dd = np.sqrt(brute.pinned_d2(p[[x]], p[[t.i64(oracle.F_VP)[a]]])[0, 0]).astype(np.float32)
                goes_in = dd <= t.f32(oracle.F_RIN)[a]
                if goes_in != (side == 0):
                    tie = side == 1 and dd == t.f32(oracle.F_RIN)[a]
                    break
            else:
                sd, sp = t.i64(oracle.F_SPLITDIM)[a], t.f32(oracle.F_SPLIT)[a]
                goes_left = p[x, sd] < sp
                if goes_left != (side == 0):
                    tie = side == 0 and p[x, sd] == sp
                    break
            v = a
        assert tie, x
        exceptions += 1
    assert exceptions < len(p) // 20
    # key order = preorder of the end node (first child before second, a node
    # before its subtree): non-decreasing preorder along the sorted keys
    srt = np.argsort(keys, kind="stable")
    assert np.all(np.diff(pre_end[srt]) >= 0)

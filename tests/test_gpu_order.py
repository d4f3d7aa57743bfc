"""Autoropes keep the recursive visit order (§3.3: "the order
that the tree is traversed is unchanged"), checked on the GPU through the
per-point visit hashes of tt_stats (include/tt.h):

  * visit_hash = h*31 + pre + 1 over the nodes a point tests, in order: equal
    to the recursive oracle's (`oracle.*(stats=True).hash`) for every
    independent walk, the per-node lockstep BH / PC walks (Fig.8 only masks)
    and the explicit rope-stack variants;
  * kNN / VP / NN lockstep lanes follow the warp's majority-vote order (§4.3):
    their hashes, visit counts and the warp's node tests equal the oracle's
    Fig.8 + majority-vote simulation;
  * the BH child-group lockstep walk and the split PC walk keep the visited
    SET (reading R23): visit_set equals the oracle's set hash, visit_hash is 0.
Also: the per-node lockstep BH walks flush their fp32 partials per body
after the same number of own visits as the independent walk, so L and N
accelerations are bit-identical.
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


def dev(a, dtype=torch.float32):
    return torch.from_numpy(np.ascontiguousarray(a)).to("cuda", dtype)


def hashes(st):
    return st.hashes()


@pytest.fixture(scope="module")
def bh():
    b = ttgen.plummer(9001, seed=401)
    b[50:53, :3] = b[7, :3]  # a depth-32 bucket
    ot = oracle.build_oct(b)
    ref = oracle.bh(ot, b, 0.5, 0.05, self_ids=np.arange(len(b)), stats=True)
    return b, ot, ref, P.tt_tree_upload(P.build_oct(b))


@pytest.fixture(scope="module")
def kd():
    p = ttgen.gaussian_mixture(12000, 7, seed=402, components=8)
    p[100:105] = p[3]
    q = np.concatenate([ttgen.gaussian_mixture(3001, 7, seed=403, components=8), p[:40]])
    ot = oracle.build_kd(p, 8)
    return p, q, ot, P.tt_tree_upload(P.build_kd(p, 8))


@pytest.mark.parametrize("variant,mode", [("autoropes", "independent"), ("ropes", "independent"),
                                          ("ropes", "lockstep"), ("stack", "independent"),
                                          ("stack", "lockstep"), ("recursive", "independent")])
@pytest.mark.parametrize("sorted_", [False, True])
def test_bh_order_hash(bh, variant, mode, sorted_):
    b, ot, ref, tree = bh
    bd = dev(b)
    order = P.tt_sort_points(tree, bd) if sorted_ else None
    st = P.Stats.alloc(len(b), "cuda", hashes=True)
    P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=order, mode=mode, stats=st, variant=variant)
    h, s = hashes(st)
    assert np.array_equal(st.visits.cpu().numpy(), ref.visits)
    assert np.array_equal(h, ref.hash)
    assert np.array_equal(s, ref.set_hash)


@pytest.mark.parametrize("sorted_", [False, True])
def test_bh_group_walk_keeps_the_visited_set(bh, sorted_):
    """Child-group lockstep tiles test each body's recursive node SET in
    DFS-over-groups order (reading R23): set hashes equal, order slot 0;
    AUTO's independent tiles keep the order."""
    b, ot, ref, tree = bh
    bd = dev(b)
    order = P.tt_sort_points(tree, bd) if sorted_ else None
    for mode in ("lockstep", "auto"):
        st = P.Stats.alloc(len(b), "cuda", hashes=True)
        P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=order, mode=mode, stats=st)
        h, s = hashes(st)
        assert np.array_equal(s, ref.set_hash)
        o = order.cpu().numpy() if sorted_ else np.arange(len(b))
        T = 32 * P._lib.BH_POINTS_PER_LANE
        wm = st.warp_mode.cpu().numpy()[:(len(b) + T - 1) // T]
        lock_pt = np.zeros(len(b), bool)
        lock_pt[o] = np.repeat(wm == 1, T)[:len(b)]
        assert np.all(h[lock_pt] == 0)
        assert np.array_equal(h[~lock_pt], ref.hash[~lock_pt])
        if mode == "lockstep":
            assert lock_pt.all()


@pytest.mark.parametrize("variant", ["ropes", "stack"])
@pytest.mark.parametrize("sorted_", [False, True])
def test_bh_per_node_lockstep_bit_identical_to_independent(bh, variant, sorted_):
    """Fig.8 only masks: the per-node lockstep walk adds, per body, the same
    terms in the same order as the independent walk and flushes its fp32
    partials after the same number of own visits -> identical bits."""
    b, ot, ref, tree = bh
    bd = dev(b)
    order = P.tt_sort_points(tree, bd) if sorted_ else None
    a_l = P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=order, mode="lockstep", variant=variant).cpu().numpy()
    a_n = P.tt_traverse_bh(tree, bd, 0.5, 0.05, order=order, mode="independent", variant=variant).cpu().numpy()
    assert np.array_equal(a_l, a_n)


@pytest.mark.parametrize("variant,mode", [("autoropes", "independent"), ("autoropes", "lockstep"),
                                          ("stack", "independent"), ("stack", "lockstep"),
                                          ("recursive", "independent"), ("split", "auto")])
def test_pc_order_hash(variant, mode):
    p = ttgen.uniform(6000, 3, seed=404)
    p[10:14] = p[2]
    ot = oracle.build_kd(p, 1)
    ref = oracle.pc(ot, p, 0.1, stats=True)
    tree = P.tt_tree_upload(P.build_kd(p, 1))
    pd = dev(p)
    for order in (None, P.tt_sort_points(tree, pd)):
        st = P.Stats.alloc(len(p), "cuda", hashes=True, point_tests=True)
        cnt = P.tt_traverse_pc(tree, pd, 0.1, order=order, mode=mode, stats=st, variant=variant)
        h, s = hashes(st)
        assert np.array_equal(cnt.cpu().numpy().astype(np.uint32), ref.out[0])
        assert np.array_equal(st.visits.cpu().numpy(), ref.visits)
        assert np.array_equal(s, ref.set_hash)
        if variant == "split":
            assert np.all(h == 0)
        else:
            assert np.array_equal(h, ref.hash)
        # leaf size 1: every untruncated leaf tests its one point, and it is
        # counted iff within r -- so tests >= count
        assert np.all(st.point_tests.cpu().numpy() >= ref.out[0])


@pytest.mark.parametrize("variant", ["autoropes", "recursive"])
def test_knn_independent_order_hash(kd, variant):
    p, q, ot, tree = kd
    ref = oracle.knn(ot, q, 8, stats=True)
    st = P.Stats.alloc(len(q), "cuda", hashes=True, point_tests=True)
    idx, d2 = P.tt_traverse_knn(tree, dev(q), 8, mode="independent", stats=st, variant=variant)
    h, s = hashes(st)
    assert np.array_equal(idx.cpu().numpy(), ref.out[0])
    assert np.array_equal(h, ref.hash) and np.array_equal(s, ref.set_hash)
    assert np.all(st.point_tests.cpu().numpy() >= 8)


@pytest.mark.parametrize("sorted_", [False, True])
def test_knn_lockstep_lanes_follow_the_majority_vote_simulation(kd, sorted_):
    p, q, ot, tree = kd
    qd = dev(q)
    order = P.tt_sort_points(tree, qd) if sorted_ else None
    o = order.cpu().numpy() if sorted_ else np.arange(len(q))
    sim = oracle.knn_lockstep(ot, q[o], 8)
    st = P.Stats.alloc(len(q), "cuda", hashes=True)
    P.tt_traverse_knn(tree, qd, 8, order=order, mode="lockstep", stats=st)
    h, s = hashes(st)
    assert np.array_equal(st.visits.cpu().numpy()[o], sim.lane_visits)
    assert np.array_equal(h[o], sim.lane_hash)
    assert np.array_equal(st.warp_fetches.cpu().numpy(), sim.warp_fetches)
    assert np.array_equal(st.warp_steps.cpu().numpy(), sim.warp_tests)  # nodes the warp tested


@pytest.fixture(scope="module")
def vp16():
    p = ttgen.gaussian_mixture(8000, 16, seed=405, components=6)
    p[70:73] = p[1]
    q = np.concatenate([ttgen.gaussian_mixture(1501, 16, seed=406, components=6), p[:20]])
    return p, q, oracle.build_vp(p), P.tt_tree_upload(P.build_vp(p))


@pytest.mark.parametrize("mode", ["independent", "lockstep"])
@pytest.mark.parametrize("sorted_", [False, True])
def test_vp_order_hash(vp16, mode, sorted_):
    p, q, ot, tree = vp16
    qd = dev(q)
    order = P.tt_sort_points(tree, qd) if sorted_ else None
    st = P.Stats.alloc(len(q), "cuda", hashes=True)
    idx, d2 = P.tt_traverse_vp(tree, qd, order=order, mode=mode, stats=st)
    h, s = hashes(st)
    if mode == "independent":
        ref = oracle.vp(ot, q, stats=True)
        assert np.array_equal(h, ref.hash) and np.array_equal(s, ref.set_hash)
        st2 = P.Stats.alloc(len(q), "cuda", hashes=True)
        P.tt_traverse_vp(tree, qd, order=order, mode=mode, stats=st2, variant="recursive")
        assert np.array_equal(hashes(st2)[0], ref.hash)
    else:
        o = order.cpu().numpy() if sorted_ else np.arange(len(q))
        sim = oracle.vp_lockstep(ot, q[o])
        assert np.array_equal(st.visits.cpu().numpy()[o], sim.lane_visits)
        assert np.array_equal(h[o], sim.lane_hash)
        assert np.array_equal(st.warp_steps.cpu().numpy(), sim.warp_tests)


@pytest.mark.parametrize("mode", ["independent", "lockstep"])
def test_nn_order_hash(mode):
    p = ttgen.gaussian_mixture(10000, 7, seed=407, components=6)
    q = ttgen.gaussian_mixture(2003, 7, seed=408, components=6)
    ot = oracle.build_nn(p)
    tree = P.tt_tree_upload(P.build_nn(p))
    qd = dev(q)
    order = P.tt_sort_points(tree, qd)
    st = P.Stats.alloc(len(q), "cuda", hashes=True)
    P.tt_traverse_nn(tree, qd, order=order, mode=mode, stats=st)
    h, s = hashes(st)
    if mode == "independent":
        ref = oracle.nn(ot, q, stats=True)
        assert np.array_equal(h, ref.hash) and np.array_equal(s, ref.set_hash)
    else:
        o = order.cpu().numpy()
        sim = oracle.nn_lockstep(ot, q[o])
        assert np.array_equal(h[o], sim.lane_hash)
        assert np.array_equal(st.warp_steps.cpu().numpy(), sim.warp_tests)


def test_hash_map_on_device_built_trees():
    """The preorder map is derived from the device records, so trees built on
    the GPU (top levels renumbered level by level) hash like the oracle."""
    b = ttgen.plummer(20011, seed=409)
    ot = oracle.build_oct(b)
    ref = oracle.bh(ot, b, 0.5, 0.05, self_ids=np.arange(len(b)), stats=True)
    tree = P.tt_build_oct_device(dev(b))
    st = P.Stats.alloc(len(b), "cuda", hashes=True)
    P.tt_traverse_bh(tree, dev(b), 0.5, 0.05, mode="independent", stats=st)
    h, s = hashes(st)
    assert np.array_equal(h, ref.hash) and np.array_equal(s, ref.set_hash)
    p = ttgen.gaussian_mixture(15000, 7, seed=410, components=6)
    kt = P.tt_build_kd_device(dev(p), 8)
    refk = oracle.knn(oracle.build_kd(p, 8), p[:3000], 8, stats=True)
    st = P.Stats.alloc(3000, "cuda", hashes=True)
    P.tt_traverse_knn(kt, dev(p[:3000]), 8, mode="independent", stats=st)
    assert np.array_equal(hashes(st)[0], refk.hash)

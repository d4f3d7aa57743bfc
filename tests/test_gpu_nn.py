"""GPU parity of the NEXT-3 NN kernel (point-per-node kd-tree, the paper's NN
benchmark P:L1216-1219, reading R21) against the CPU oracle, through the C
ABI: indices and d2 bit-exact, per-point visit counts exact in independent
mode (autoropes keep the recursive order), lockstep warp fetches
and lane visits equal the oracle's Fig.8 + majority-vote simulation."""
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


def dev(a, dtype=torch.float32):
    return torch.from_numpy(np.ascontiguousarray(a)).to("cuda", dtype)


@pytest.fixture(scope="module", params=[7, 16, 3])
def nn_small(request):
    dim = request.param
    p = ttgen.gaussian_mixture(20011, dim, seed=300 + dim, components=16)
    p[100:105] = p[7]  # exact duplicates: ties broken by id
    q = np.concatenate([ttgen.gaussian_mixture(4000, dim, seed=400 + dim, components=16), p[:37]])
    ot = oracle.build_nn(p)
    tree = P.tt_tree_upload(P.build_nn(p))
    return p, q, ot, tree


def test_nn_independent_bit_exact_and_visits(nn_small):
    p, q, ot, tree = nn_small
    ref = oracle.nn(ot, q, stats=True)
    st = P.Stats.alloc(len(q), "cuda")
    idx, d2 = P.tt_traverse_nn(tree, dev(q), mode="independent", stats=st)
    assert np.array_equal(idx.cpu().numpy(), ref.out[0])
    assert np.array_equal(d2.cpu().numpy(), ref.out[1])
    assert np.array_equal(st.visits.cpu().numpy(), ref.visits)


@pytest.mark.parametrize("sorted_", [False, True])
def test_nn_lockstep_matches_simulation(nn_small, sorted_):
    p, q, ot, tree = nn_small
    qd = dev(q)
    order = P.tt_sort_points(tree, qd) if sorted_ else None
    o = order.cpu().numpy() if sorted_ else np.arange(len(q))
    li, ld, lv, wf = oracle.nn_lockstep(ot, q[o])
    st = P.Stats.alloc(len(q), "cuda")
    idx, d2 = P.tt_traverse_nn(tree, qd, order=order, mode="lockstep", stats=st)
    assert np.array_equal(idx.cpu().numpy()[o], li) and np.array_equal(d2.cpu().numpy()[o], ld)
    assert np.array_equal(st.visits.cpu().numpy()[o], lv)
    assert np.array_equal(st.warp_fetches.cpu().numpy(), wf)


@pytest.mark.parametrize("mode", MODES)
def test_nn_every_mode_equals_bruteforce_definition(nn_small, mode):
    p, q, ot, tree = nn_small
    ref = oracle.nn(ot, q)
    qd = dev(q)
    for order in (None, P.tt_sort_points(tree, qd)):
        if order is not None:
            order = P.tt_schedule_tiles(tree, qd, order)
        idx, d2 = P.tt_traverse_nn(tree, qd, order=order, mode=mode)
        assert np.array_equal(idx.cpu().numpy(), ref.out[0]) and np.array_equal(d2.cpu().numpy(), ref.out[1])


def test_nn_sort_keys_match_oracle(nn_small):
    p, q, ot, tree = nn_small
    keys = torch.empty(len(q), dtype=torch.int64, device="cuda")
    perm = P.tt_sort_points(tree, dev(q), keys=keys)
    assert np.array_equal(keys.cpu().numpy().view(np.uint64), oracle.sort_keys(ot, q))
    assert np.array_equal(perm.cpu().numpy(), oracle.sort_perm(ot, q))


def test_nn_edges():
    p = ttgen.gaussian_mixture(500, 7, seed=310, components=4)
    ot = oracle.build_nn(p)
    tree = P.tt_tree_upload(P.build_nn(p))
    idx, d2 = P.tt_traverse_nn(tree, dev(p[:0]))
    assert idx.numel() == 0
    for n in (1, 7, 31, 33):
        for mode in MODES:
            idx, d2 = P.tt_traverse_nn(tree, dev(p[:n] + 0.001), mode=mode)
            ri, rd = oracle.nn(ot, p[:n] + np.float32(0.001)).out
            assert np.array_equal(idx.cpu().numpy(), ri) and np.array_equal(d2.cpu().numpy(), rd)
    one = ttgen.gaussian_mixture(1, 7, seed=311, components=1)
    t1 = P.tt_tree_upload(P.build_nn(one))
    idx, d2 = P.tt_traverse_nn(t1, dev(p[:40]))
    assert np.all(idx.cpu().numpy() == 0)
    with pytest.raises(P.TTError):
        P.tt_traverse_vp(tree, dev(p[:4]))  # kind mismatch


@pytest.mark.slow
def test_nn_1m_sampled():
    c = ttgen.CONFIGS["knn_1m_7d"]
    p = ttgen.gaussian_mixture(c["n"], c["dim"], c["seed"])
    q = ttgen.gaussian_mixture(c["m"], c["dim"], c["qseed"])
    tree = P.tt_tree_upload(P.build_nn(p))
    qd = dev(q)
    perm = P.tt_schedule_tiles(tree, qd, P.tt_sort_points(tree, qd))
    idx, d2 = P.tt_traverse_nn(tree, qd, order=perm)
    sample = np.random.default_rng(3).choice(len(q), 2000, replace=False)
    ref = oracle.nn(oracle.build_nn(p), q[sample])
    assert np.array_equal(idx.cpu().numpy()[sample], ref.out[0])
    assert np.array_equal(d2.cpu().numpy()[sample], ref.out[1])


@pytest.mark.parametrize("n,dim", [(1, 3), (2, 3), (3, 2), (7, 7), (5_000, 16), (20_011, 7), (1_000_000, 7)])
def test_gpu_nn_build_is_byte_identical_to_host_pack(n, dim):
    """tt_build_nn_device writes the same blob bytes as tt_tree_pack of the
    host builder (duplicates included: ties broken by id)."""
    p = ttgen.gaussian_mixture(n, dim, seed=320, components=6)
    if n > 100:
        p[50:60] = p[7]
    host_blob = P.build_nn(p).pack()
    t = P.tt_build_nn_device(dev(p))
    gpu_blob = P.tt_tree_download(t)
    assert gpu_blob.size == host_blob.size
    diff = np.nonzero(gpu_blob != host_blob)[0]
    assert diff.size == 0, f"{diff.size} bytes differ, first at {diff[:8]}"

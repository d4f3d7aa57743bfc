"""Host-side product logic, no GPU needed: the C ABI exports, the host tree
builders (parity with the oracle's independent builders, bit for bit), the
packed device layout, and argument errors.  Nothing here launches a kernel."""
from __future__ import annotations

import ctypes as C
import os
import re

import numpy as np
import pytest
import torch

import oracle
import ttgen
import paper_conf_sc_goldfarbjk13_b200 as P
from paper_conf_sc_goldfarbjk13_b200 import _lib as L

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_library_exports_every_declared_symbol():
    hdr = open(os.path.join(ROOT, "include", "tt.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)
    declared = set(re.findall(r"\b(tt_[a-z_0-9]+)\s*\(", hdr))
    assert len(declared) >= 24
    lib = C.CDLL(L.LIB_PATH)
    for name in sorted(declared):
        assert hasattr(lib, name), name
    assert declared == set(L.SIGNATURES), declared ^ set(L.SIGNATURES)


def test_build_info_names_sm100a():
    assert "sm_100a" in P.build_info()


# --------------------------------------------------------- builder parity
@pytest.mark.parametrize("n,dim,leaf", [(3000, 3, 1), (4000, 7, 8), (1000, 16, 4)])
def test_kd_builder_matches_oracle(n, dim, leaf):
    p = ttgen.gaussian_mixture(n, dim, seed=101, components=5)
    p[::97] = p[1]
    h, o = P.build_kd(p, leaf), oracle.build_kd(p, leaf)
    assert h.n_nodes == o.n_nodes and h.height == o.height
    for name, f in [("skip", oracle.F_SKIP), ("level", oracle.F_LEVEL), ("pbegin", oracle.F_PBEGIN),
                    ("pcount", oracle.F_PCOUNT), ("split_dim", oracle.F_SPLITDIM)]:
        assert np.array_equal(h.array(name), o.i64(f)), name
    assert np.array_equal(h.array("split"), o.f32(oracle.F_SPLIT))
    assert np.array_equal(h.array("lo"), o.f32(oracle.F_LO, dim))
    assert np.array_equal(h.array("hi"), o.f32(oracle.F_HI, dim))
    assert np.array_equal(h.array("tree_order"), o.tree_order())
    fc = h.array("first_child")
    assert np.array_equal(fc, o.children()[:, 0])


def test_oct_builder_matches_oracle_bit_for_bit():
    b = ttgen.plummer(20000, seed=102)
    b[7, :3] = b[8, :3]  # exercise the depth-32 bucket
    h, o = P.build_oct(b), oracle.build_oct(b)
    assert h.n_nodes == o.n_nodes and h.height == o.height == 33
    assert np.array_equal(h.array("skip"), o.i64(oracle.F_SKIP))
    assert np.array_equal(h.array("level"), o.i64(oracle.F_LEVEL))
    assert np.array_equal(h.array("body"), o.i64(oracle.F_BODY))
    com = h.array("com")
    for c, f in enumerate([oracle.F_COMX, oracle.F_COMY, oracle.F_COMZ, oracle.F_MASS]):
        assert np.array_equal(com[:, c], o.f32(f))
    assert np.array_equal(h.array("tree_order"), o.tree_order())
    c, s = o.root_cube()
    hc, hs = h.root_cube
    assert np.array_equal(c, hc) and s == hs


def test_vp_builder_matches_oracle():
    p = ttgen.gaussian_mixture(3000, 16, seed=103, components=4)
    p[10:13] = p[50]
    h, o = P.build_vp(p), oracle.build_vp(p)
    assert h.n_nodes == o.n_nodes == 3000 and h.height == o.height
    assert np.array_equal(h.array("body"), o.i64(oracle.F_VP))
    assert np.array_equal(h.array("r_in_max"), o.f32(oracle.F_RIN))
    assert np.array_equal(h.array("r_out_min"), o.f32(oracle.F_ROUT))
    ch = o.children()
    assert np.array_equal(h.array("in_child"), ch[:, 0])
    assert np.array_equal(h.array("out_child"), ch[:, 1])
    assert np.array_equal(h.array("skip"), o.i64(oracle.F_SKIP))


@pytest.mark.parametrize("n,dim", [(3001, 7), (1, 3), (2, 16), (700, 2)])
def test_nn_builder_matches_oracle(n, dim):
    """NEXT-3 point-per-node kd-tree (R21): libtt's builder vs the oracle's."""
    p = ttgen.gaussian_mixture(n, dim, seed=105, components=4)
    if n > 100:
        p[20:25] = p[60]
    h, o = P.build_nn(p), oracle.build_nn(p)
    assert h.kind == "nn" and h.n_nodes == o.n_nodes == n and h.height == o.height
    assert np.array_equal(h.array("body"), o.i64(oracle.F_VP))
    assert np.array_equal(h.array("split_dim"), o.i64(oracle.F_SPLITDIM))
    sd = o.i64(oracle.F_SPLITDIM) >= 0
    assert np.array_equal(h.array("split")[sd], o.f32(oracle.F_SPLIT)[sd])
    ch = o.children()
    assert np.array_equal(h.array("in_child"), ch[:, 0])
    assert np.array_equal(h.array("out_child"), ch[:, 1])
    assert np.array_equal(h.array("skip"), o.i64(oracle.F_SKIP))
    assert np.array_equal(h.array("level"), o.i64(oracle.F_LEVEL))
    assert np.array_equal(h.array("tree_order"), o.tree_order())
    assert np.array_equal(h.array("lo"), o.f32(oracle.F_LO, dim).reshape(-1, dim))
    assert np.array_equal(h.array("hi"), o.f32(oracle.F_HI, dim).reshape(-1, dim))


def test_nn_blob_records_and_points():
    p = ttgen.gaussian_mixture(2500, 7, seed=106, components=4)
    h = P.build_nn(p)
    blob = h.pack()
    hd = {k: (int(v) if np.ndim(v) == 0 else v) for k, v in
          zip(HDR.names, np.frombuffer(blob[:HDR.itemsize].tobytes(), HDR)[0])}
    assert hd["kind"] == 4 and hd["rec_bytes"] == 16 and hd["dp"] == 8 and hd["n_nodes"] == 2500
    N = h.n_nodes
    rec = np.frombuffer(blob[hd["off_rec"]:hd["off_rec"] + 16 * N].tobytes(),
                        dtype=[("l", "<i4"), ("r", "<i4"), ("split", "<f4"), ("dim", "<i4")])
    pts = np.frombuffer(blob[hd["off_vpt"]:hd["off_vpt"] + 32 * N].tobytes(), "<f4").reshape(N, 8)
    pid = np.frombuffer(blob[hd["off_pid"]:hd["off_pid"] + 4 * N].tobytes(), "<i4")
    assert np.array_equal(np.sort(pid), np.arange(N))
    assert np.array_equal(pts[:, :7], p[pid]) and np.all(pts[:, 7] == 0)
    box = np.frombuffer(blob[hd["off_box"]:hd["off_box"] + 64 * N].tobytes(), "<f4").reshape(N, 2, 8)
    # subtree point sets from the device numbering; every node's box is their
    # tight box and every child satisfies the node's split rule
    def subtree(v):
        out, st = [], [v]
        while st:
            u = st.pop()
            out.append(u)
            st += [c for c in (rec["l"][u], rec["r"][u]) if c >= 0]
        return out
    seen = 0
    for v in range(N):
        ids = pid[subtree(v)]
        assert np.array_equal(box[v, 0, :7], p[ids].min(0)) and np.array_equal(box[v, 1, :7], p[ids].max(0))
        for c, side in ((rec["l"][v], 0), (rec["r"][v], 1)):
            if c < 0:
                continue
            d = rec["dim"][v]
            assert d >= 0
            assert (p[pid[c], d] <= rec["split"][v]) if side == 0 else (p[pid[c], d] >= rec["split"][v])
        seen += 1
    assert seen == N


# ------------------------------------------------------------- blob layout
HDR = np.dtype([("magic", "<u4"), ("version", "<u4"), ("kind", "<i4"), ("dim", "<i4"), ("dp", "<i4"),
                ("height", "<i4"), ("leaf_size", "<i4"), ("top_levels", "<i4"), ("top_count", "<i4"),
                ("oct_flags", "<i4"), ("level_prefix", "<i4", 33), ("pad1", "<i4"), ("n_nodes", "<i8"), ("n_points", "<i8"), ("root_center", "<f8", 3),
                ("root_side", "<f8"), ("off_rec", "<u8"), ("off_box", "<u8"), ("off_pts", "<u8"),
                ("off_pid", "<u8"), ("off_vpt", "<u8"), ("total", "<u8"), ("rec_bytes", "<u8"), ("off_cbox", "<u8")])


def _walk_preorder(first_child, skip, n):
    """Device-index sequence of a full unguided walk (never truncate)."""
    seq, cur = [], 0
    while cur != -1:
        seq.append(cur)
        cur = first_child[cur] if first_child[cur] >= 0 else skip[cur]
    return seq


def test_oct_blob_top_first_layout_preserves_preorder():
    b = ttgen.plummer(5000, seed=104)
    h = P.build_oct(b)
    blob = h.pack()
    hd = {k: (int(v) if np.ndim(v) == 0 else v) for k, v in
          zip(HDR.names, np.frombuffer(blob[:HDR.itemsize].tobytes(), HDR)[0])}
    assert hd["magic"] == 0x31425454 and hd["kind"] == 1 and hd["n_nodes"] == h.n_nodes
    assert hd["oct_flags"] == 3  # NARROW | FEW_CELL_KIDS: no depth-32 bucket
    rec = np.frombuffer(blob[hd["off_rec"]:hd["off_rec"] + 32 * h.n_nodes].tobytes(),
                        dtype=[("g", "<f4", 4), ("fc", "<i4"), ("skip", "<i4"), ("body", "<i4"), ("lvl", "<i4")])
    top = hd["top_count"]
    assert 0 < top * 32 <= 32 * 1024
    assert np.all(rec["lvl"][:top] < hd["top_levels"]) and np.all(rec["lvl"][top:] >= hd["top_levels"])
    # top region numbered level by level: every level-complete prefix is the top L levels
    assert np.all(np.diff(rec["lvl"][:top]) >= 0)
    lp = hd["level_prefix"]
    for L in range(hd["top_levels"] + 1):
        assert lp[L] == int((h.array("level") < L).sum())
    seq = _walk_preorder(rec["fc"], rec["skip"], h.n_nodes)
    assert len(seq) == h.n_nodes and len(set(seq)) == h.n_nodes
    # the walk visits nodes in canonical preorder: levels and bodies line up
    assert np.array_equal(rec["lvl"][seq], h.array("level"))
    assert np.array_equal(rec["body"][seq], h.array("body"))
    assert np.array_equal(rec["g"][seq], h.array("com"))


@pytest.mark.parametrize("dup", [2, 8, 9, 40])
def test_oct_blob_flags_for_buckets(dup):
    """A depth-32 bucket (R9) of `dup` coincident bodies: height 33, so the
    header says "not narrow" (the child-group walk stages its groups 8 at a
    time); its children are leaves, so at most 8 cell children per node."""
    b = ttgen.plummer(500, seed=106)
    b[10:10 + dup, :3] = b[3, :3]
    h = P.build_oct(b)
    blob = h.pack()
    hd = {k: (int(v) if np.ndim(v) == 0 else v) for k, v in
          zip(HDR.names, np.frombuffer(blob[:HDR.itemsize].tobytes(), HDR)[0])}
    assert hd["height"] == 33 and hd["oct_flags"] == 2


def test_kd_blob_children_and_points():
    p = ttgen.uniform(3000, 7, seed=105)
    h = P.build_kd(p, 8)
    blob = h.pack()
    hd = {k: (int(v) if np.ndim(v) == 0 else v) for k, v in
          zip(HDR.names, np.frombuffer(blob[:HDR.itemsize].tobytes(), HDR)[0])}
    dp = hd["dp"]
    assert dp == 8
    rec = np.frombuffer(blob[hd["off_rec"]:hd["off_rec"] + 32 * h.n_nodes].tobytes(),
                        dtype=[("left", "<i4"), ("right", "<i4"), ("skip", "<i4"), ("lvl", "<i4"),
                               ("split", "<f4"), ("dim", "<i4"), ("pb", "<i4"), ("pc", "<i4")])
    seq = _walk_preorder(rec["left"], rec["skip"], h.n_nodes)
    assert np.array_equal(rec["dim"][seq], h.array("split_dim"))
    assert np.array_equal(rec["pb"][seq], h.array("pbegin"))
    inner = rec["left"] >= 0
    # right child = rope of the left child
    assert np.array_equal(rec["right"][inner], rec["skip"][rec["left"][inner]])
    pts = np.frombuffer(blob[hd["off_pts"]:hd["off_pts"] + 4 * dp * 3000].tobytes(), "<f4").reshape(3000, dp)
    pid = np.frombuffer(blob[hd["off_pid"]:hd["off_pid"] + 4 * 3000].tobytes(), "<i4")
    assert np.array_equal(pid, h.array("tree_order"))
    assert np.array_equal(pts[:, :7], p[pid]) and np.all(pts[:, 7] == 0)
    box = np.frombuffer(blob[hd["off_box"]:hd["off_box"] + 8 * dp * h.n_nodes].tobytes(), "<f4")
    box = box.reshape(h.n_nodes, 2, dp)
    assert np.array_equal(box[seq, 0, :7], h.array("lo")) and np.array_equal(box[seq, 1, :7], h.array("hi"))
    # children's boxes stored with the parent (kNN layout)
    cbox = np.frombuffer(blob[hd["off_cbox"]:hd["off_cbox"] + 16 * dp * h.n_nodes].tobytes(), "<f4")
    cbox = cbox.reshape(h.n_nodes, 2, 2, dp)
    for v in np.nonzero(inner)[0][:500]:
        for c, kid in enumerate((rec["left"][v], rec["right"][v])):
            assert np.array_equal(cbox[v, c, 0], box[kid, 0]) and np.array_equal(cbox[v, c, 1], box[kid, 1])


# ------------------------------------------------------------ error paths
def test_builder_argument_errors():
    lib = L.load()
    h = C.c_void_p()
    p = np.zeros((4, 3), np.float32)
    assert lib.tt_build_kd(None, 4, 3, 3, 1, C.byref(h)) == -1
    assert lib.tt_build_kd(p.ctypes.data, 4, 3, 2, 1, C.byref(h)) == -1  # ld < dim
    assert lib.tt_build_kd(p.ctypes.data, 4, 17, 17, 1, C.byref(h)) == -1  # dim > TT_MAX_DIM
    assert lib.tt_build_kd(p.ctypes.data, 0, 3, 3, 1, C.byref(h)) == -1
    assert lib.tt_traverse_bh(None, None, None, 0, 0.5, 0.05, None, None, None) == -1
    assert lib.tt_sort_points(None, None, 0, 3, None, None, None) == -1
    assert lib.tt_status_string(-4) == b"TT_ERR_TREE_TOO_DEEP"


def test_pack_rejects_too_deep_tree():
    # a degenerate chain: duplicates of one body force a depth-32 bucket of > 8 ...
    # instead craft a kd desc whose height exceeds TT_MAX_HEIGHT
    h = P.build_kd(ttgen.uniform(64, 2, seed=106), 1)
    d = L.tt_tree_desc.from_buffer_copy(h.desc)
    d.height = L.MAX_HEIGHT + 1
    n = C.c_size_t()
    assert L.load().tt_tree_pack_size(C.byref(d), C.byref(n)) == -4


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU behaviour")
def test_no_cpu_fallback_without_gpu():
    h = P.build_kd(ttgen.uniform(100, 3, seed=107), 1)
    with pytest.raises(P.TTError) as e:
        P.tt_tree_from_blob(h.pack())
    assert e.value.status == -2  # TT_ERR_CUDA

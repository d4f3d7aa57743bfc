"""CPU oracle for the batched point-by-tree traversal (Goldfarb, Jo & Kulkarni, SC'13).

TEST INFRASTRUCTURE ONLY: only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package.  It shares no code with ``paper_conf_sc_goldfarbjk13_b200`` (the CUDA
path) and never imports it.

The arithmetic lives in ``oracle.c`` (plain recursive C, one function per
paper figure, see its header); this module only compiles it with
``-O2 -ffp-contract=off -fopenmp`` and marshals numpy arrays through ctypes.

Parity status of each function:
  build_kd / build_oct / build_vp  pinned: invariants + brute-force partition checks; oct
                                   buckets of any size (R9) == direct sum at theta = 0
  linearise (skip/preorder)        pinned: Fig.2 worked example (tests/golden/fig2_ropes.txt)
  pc                               pinned: all-pairs brute force, symmetry, r=inf
  bh                               pinned: theta=0 == O(n^2) direct sum, two-body closed form,
                                   the R8 opening test by a hand-worked 10-node example
                                   (visits, order hash, forces), error monotone in theta;
                                   1M-Plummer visits/body and work expansion within 10% of
                                   Tables 1-2 (sanity)
  knn                              pinned: brute-force partial sort on (d2, id)
  vp                               pinned: brute-force argmin on (d2, id)
  build_nn / nn (NEXT-3, R21)      pinned: brute-force argmin on (d2, id), == kNN k=1 == VP;
                                   builder: median/split/partition invariants
  sort_keys                        pinned: kd/oct Morton/preorder invariants; vp/nn: a data
                                   point's descent passes its own node except at checked
                                   boundary ties; keys sort in preorder of the end node
  visit hashes (stats=True)        pinned: order hash of a full walk == preorder sequence; set
                                   hash == sum over all nodes; R8 example's order hash
  *_lockstep, unguided_warp_union  pinned: results == independent walks; per warp, nodes tested
                                   >= the longest lane; Table 2 work expansion >= 1 on average
                                   (P:L2307-2313); a one-lane warp == the recursive walk;
                                   absolute fetch counts on our inputs: parity unpinned
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

F_LEVEL, F_SKIP, F_NCHILD, F_PBEGIN, F_PCOUNT, F_LABEL = 0, 1, 2, 3, 4, 5
F_CHILD0 = 10
F_SPLITDIM, F_BODY, F_VP = 20, 21, 22
F_SPLIT, F_MASS, F_COMX, F_COMY, F_COMZ, F_RIN, F_ROUT = 40, 41, 42, 43, 44, 45, 46
F_LO, F_HI = 60, 61


def build(force: bool = False) -> str:
    """Compile liboracle.so (gcc, no fast-math, no FMA contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-std=c11", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
               "-fPIC", "-shared", "-Wall", "-o", _LIB + ".tmp", _SRC, "-lm"]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(_LIB)
        P, I64, I, F = C.c_void_p, C.c_int64, C.c_int, C.c_float
        L.or_build_kd.restype = P
        L.or_build_kd.argtypes = [P, I64, I, I, I]
        L.or_build_oct.restype = P
        L.or_build_oct.argtypes = [P, I64]
        L.or_build_vp.restype = P
        L.or_build_vp.argtypes = [P, I64, I, I]
        L.or_build_nn.restype = P
        L.or_build_nn.argtypes = [P, I64, I, I]
        L.or_build_generic.restype = P
        L.or_build_generic.argtypes = [I, P, P, I]
        L.or_free.argtypes = [P]
        L.or_num_nodes.restype = I64
        L.or_num_nodes.argtypes = [P]
        L.or_height.restype = I
        L.or_height.argtypes = [P]
        L.or_root_cube.argtypes = [P, P, P]
        L.or_export_i64.argtypes = [P, I, P]
        L.or_export_f32.argtypes = [P, I, P]
        L.or_tree_order.argtypes = [P, P]
        L.or_pc.argtypes = [P, P, I64, I, F, P, P, P, P, I]
        L.or_bh_dsq_root.restype = F
        L.or_bh_dsq_root.argtypes = [P, F]
        L.or_bh.argtypes = [P, P, P, I64, F, F, P, P, P, P, I]
        L.or_knn.argtypes = [P, P, I64, I, I, P, P, P, P, P, I]
        L.or_vp.argtypes = [P, P, I64, I, P, P, P, P, P, I]
        L.or_sort_keys.argtypes = [P, P, I64, I, P, I]
        L.or_unguided_warp_union.argtypes = [P, P, I64, I, I, F, P, I]
        L.or_knn_lockstep.argtypes = [P, P, I64, I, I, P, P, P, P, P, P, I]
        L.or_vp_lockstep.argtypes = [P, P, I64, I, P, P, P, P, P, P, I]
        L.or_nn.argtypes = [P, P, I64, I, P, P, P, P, P, I]
        L.or_nn_lockstep.argtypes = [P, P, I64, I, P, P, P, P, P, P, I]
        L.or_max_threads.restype = I
        _lib = L
    return _lib


def max_threads() -> int:
    return int(lib().or_max_threads())


def _p(a: np.ndarray | None):
    return None if a is None else a.ctypes.data


def _f32(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float32)


class Tree:
    """An oracle tree (pointer-style in C) plus views of its preorder export."""

    def __init__(self, handle, kind: str, pts: np.ndarray):
        if not handle:
            raise ValueError("oracle tree build failed")
        self._h = handle
        self.kind = kind
        self.pts = pts  # keep the caller's points alive (the C tree points into them)
        self.n_nodes = int(lib().or_num_nodes(handle))
        self.height = int(lib().or_height(handle))

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.or_free(self._h)
            self._h = None

    def i64(self, field: int) -> np.ndarray:
        out = np.empty(self.n_nodes, dtype=np.int64)
        if lib().or_export_i64(self._h, field, _p(out)) != 0:
            raise ValueError(field)
        return out

    def f32(self, field: int, width: int = 1) -> np.ndarray:
        out = np.empty(self.n_nodes * width, dtype=np.float32)
        if lib().or_export_f32(self._h, field, _p(out)) != 0:
            raise ValueError(field)
        return out.reshape(self.n_nodes, width) if width > 1 else out

    def children(self) -> np.ndarray:
        return np.stack([self.i64(F_CHILD0 + c) for c in range(8)], axis=1)

    def tree_order(self) -> np.ndarray:
        out = np.empty(len(self.pts), dtype=np.int64)
        lib().or_tree_order(self._h, _p(out))
        return out

    def root_cube(self):
        c = np.zeros(3, dtype=np.float64)
        s = np.zeros(1, dtype=np.float64)
        lib().or_root_cube(self._h, _p(c), _p(s))
        return c, float(s[0])


def build_kd(pts: np.ndarray, leaf_size: int) -> Tree:
    pts = _f32(pts)
    n, d = pts.shape
    return Tree(lib().or_build_kd(_p(pts), n, d, d, leaf_size), "kd", pts)


def build_oct(bodies: np.ndarray) -> Tree:
    b = _f32(bodies)
    assert b.ndim == 2 and b.shape[1] == 4
    return Tree(lib().or_build_oct(_p(b), len(b)), "oct", b)


def build_vp(pts: np.ndarray) -> Tree:
    pts = _f32(pts)
    n, d = pts.shape
    return Tree(lib().or_build_vp(_p(pts), n, d, d), "vp", pts)


def build_nn(pts: np.ndarray) -> Tree:
    """Point-per-node kd-tree of the paper's NN benchmark (reading R21)."""
    pts = _f32(pts)
    n, d = pts.shape
    return Tree(lib().or_build_nn(_p(pts), n, d, d), "nn", pts)


def build_generic(children: list[list[int]], root: int = 0) -> Tree:
    """Hand-given tree: children[v] = ordered child labels of node v."""
    ptr = np.zeros(len(children) + 1, dtype=np.int32)
    for v, ch in enumerate(children):
        ptr[v + 1] = ptr[v] + len(ch)
    idx = np.array([c for ch in children for c in ch] or [0], dtype=np.int32)
    h = lib().or_build_generic(len(children), _p(ptr), _p(idx), root)
    return Tree(h, "generic", np.zeros((0, 1), np.float32))


def _threads(t):
    return max_threads() if t is None else int(t)


@dataclass
class Result:
    out: tuple
    visits: np.ndarray | None = None
    hash: np.ndarray | None = None       # order-sensitive: h = h*31 + pre + 1
    set_hash: np.ndarray | None = None   # order-insensitive: sum of mix64(pre + 1)


def pc(tree: Tree, q: np.ndarray, radius: float, threads=None, stats=False) -> Result:
    q = _f32(q)
    m = len(q)
    cnt = np.empty(m, np.uint32)
    v = np.empty(m, np.int64) if stats else None
    h = np.empty(m, np.uint64) if stats else None
    sh = np.empty(m, np.uint64) if stats else None
    rc = lib().or_pc(tree._h, _p(q), m, q.shape[1], float(radius), _p(cnt), _p(v), _p(h), _p(sh), _threads(threads))
    assert rc == 0
    return Result((cnt,), v, h, sh)


def bh_dsq_root(tree: Tree, theta: float) -> float:
    return float(lib().or_bh_dsq_root(tree._h, float(theta)))


def bh(tree: Tree, bodies: np.ndarray, theta: float, eps: float, self_ids=None,
       threads=None, stats=False) -> Result:
    b = _f32(bodies)
    m = len(b)
    acc = np.empty((m, 3), np.float64)
    sid = None if self_ids is None else np.ascontiguousarray(self_ids, dtype=np.int64)
    v = np.empty(m, np.int64) if stats else None
    h = np.empty(m, np.uint64) if stats else None
    sh = np.empty(m, np.uint64) if stats else None
    rc = lib().or_bh(tree._h, _p(b), _p(sid), m, float(theta), float(eps), _p(acc), _p(v), _p(h), _p(sh),
                     _threads(threads))
    assert rc == 0
    return Result((acc,), v, h, sh)


def knn(tree: Tree, q: np.ndarray, k: int, threads=None, stats=False) -> Result:
    q = _f32(q)
    m = len(q)
    idx = np.empty((m, k), np.int64)
    d2 = np.empty((m, k), np.float32)
    v = np.empty(m, np.int64) if stats else None
    h = np.empty(m, np.uint64) if stats else None
    sh = np.empty(m, np.uint64) if stats else None
    rc = lib().or_knn(tree._h, _p(q), m, q.shape[1], k, _p(idx), _p(d2), _p(v), _p(h), _p(sh), _threads(threads))
    assert rc == 0
    return Result((idx, d2), v, h, sh)


def vp(tree: Tree, q: np.ndarray, threads=None, stats=False) -> Result:
    q = _f32(q)
    m = len(q)
    idx = np.empty(m, np.int64)
    d2 = np.empty(m, np.float32)
    v = np.empty(m, np.int64) if stats else None
    h = np.empty(m, np.uint64) if stats else None
    sh = np.empty(m, np.uint64) if stats else None
    rc = lib().or_vp(tree._h, _p(q), m, q.shape[1], _p(idx), _p(d2), _p(v), _p(h), _p(sh), _threads(threads))
    assert rc == 0
    return Result((idx, d2), v, h, sh)


def nn(tree: Tree, q: np.ndarray, threads=None, stats=False) -> Result:
    """Nearest neighbour over the R21 point-per-node kd-tree (Fig.5 pattern)."""
    q = _f32(q)
    m = len(q)
    idx = np.empty(m, np.int64)
    d2 = np.empty(m, np.float32)
    v = np.empty(m, np.int64) if stats else None
    h = np.empty(m, np.uint64) if stats else None
    sh = np.empty(m, np.uint64) if stats else None
    rc = lib().or_nn(tree._h, _p(q), m, q.shape[1], _p(idx), _p(d2), _p(v), _p(h), _p(sh), _threads(threads))
    assert rc == 0
    return Result((idx, d2), v, h, sh)


def sort_keys(tree: Tree, q: np.ndarray, threads=None) -> np.ndarray:
    q = _f32(q)
    keys = np.empty(len(q), np.uint64)
    rc = lib().or_sort_keys(tree._h, _p(q), len(q), q.shape[1], _p(keys), _threads(threads))
    assert rc == 0
    return keys


def sort_perm(tree: Tree, q: np.ndarray, threads=None) -> np.ndarray:
    """perm[j] = original index of the j-th point in tree order (stable)."""
    return np.argsort(sort_keys(tree, q, threads), kind="stable")


def unguided_warp_union(tree: Tree, pts_in_warp_order: np.ndarray, param: float, W: int = 32,
                        threads=None) -> np.ndarray:
    """Lockstep node fetches per warp for BH (param=theta) or PC (param=radius)."""
    p = _f32(pts_in_warp_order)
    nw = (len(p) + W - 1) // W
    out = np.empty(nw, np.int64)
    rc = lib().or_unguided_warp_union(tree._h, _p(p), len(p), p.shape[1], W, float(param), _p(out),
                                      _threads(threads))
    assert rc == 0
    return out


@dataclass
class LockstepResult:
    """Guided lockstep simulation (Fig.8 + the §4.3 majority vote).

    out: per-lane results; lane_visits / lane_hash: nodes each lane tested
    and their order hash; warp_tests: nodes each warp tested (pops, Table 2's
    numerator); warp_fetches: pops with an active lane (nodes
    expanded; reading R22)."""
    out: tuple
    lane_visits: np.ndarray
    lane_hash: np.ndarray
    warp_tests: np.ndarray
    warp_fetches: np.ndarray

    def __iter__(self):  # (idx, d2, lane_visits, warp_fetches), the round-1 tuple
        return iter((*self.out, self.lane_visits, self.warp_fetches))

    def __getitem__(self, i):
        return tuple(self)[i]


def _lockstep(fn, tree, q, k=None, threads=None):
    q = _f32(q)
    m = len(q)
    shape = (m, k) if k is not None else (m,)
    idx = np.empty(shape, np.int64)
    d2 = np.empty(shape, np.float32)
    lv = np.empty(m, np.int64)
    lh = np.empty(m, np.uint64)
    nw = (m + 31) // 32
    wf = np.empty(nw, np.int64)
    wt = np.empty(nw, np.int64)
    args = [tree._h, _p(q), m, q.shape[1]] + ([k] if k is not None else [])
    rc = fn(*args, _p(idx), _p(d2), _p(lv), _p(wf), _p(wt), _p(lh), _threads(threads))
    assert rc == 0
    return LockstepResult((idx, d2), lv, lh, wt, wf)


def knn_lockstep(tree: Tree, q: np.ndarray, k: int, threads=None) -> LockstepResult:
    return _lockstep(lib().or_knn_lockstep, tree, q, k, threads)


def vp_lockstep(tree: Tree, q: np.ndarray, threads=None) -> LockstepResult:
    return _lockstep(lib().or_vp_lockstep, tree, q, None, threads)


def nn_lockstep(tree: Tree, q: np.ndarray, threads=None) -> LockstepResult:
    return _lockstep(lib().or_nn_lockstep, tree, q, None, threads)


def work_expansion(warp_nodes: np.ndarray, independent_visits: np.ndarray, W: int = 32) -> np.ndarray:
    """Table 2's metric per warp: nodes the warp accesses in
    the lockstep traversal / nodes of its longest non-lockstep traversal.
    independent_visits: per-point N-mode visit counts in warp order."""
    v = np.asarray(independent_visits, np.float64)
    nw = len(warp_nodes)
    pad = nw * W - len(v)
    longest = np.concatenate([v, np.zeros(pad)]).reshape(nw, W).max(1)
    return np.asarray(warp_nodes, np.float64) / longest

"""Python binding of libtt (include/tt.h): same names, argument marshalling only.

Every step of the traversal path runs in libtt's CUDA kernels; PyTorch only
supplies device memory and the current stream.  There is no CPU fallback:
calls on a machine without a CUDA device raise ``TTError(TT_ERR_CUDA)``.

    host = build_oct(bodies_np)                 # tt_build_oct   (host C++ builder)
    tree = tt_tree_upload(host)                 # a0: pack + H2D
    perm = tt_sort_points(tree, bodies_dev)     # a1: keys + radix sort
    acc  = tt_traverse_bh(tree, bodies_dev, theta, eps, order=perm)   # a2-a5
"""
from __future__ import annotations

import ctypes as C
from dataclasses import dataclass

import numpy as np
import torch

from . import _lib as L
from ._lib import TTError, check

__all__ = [
    "HostTree", "Tree", "Stats", "TTError",
    "build_kd", "build_oct", "build_vp", "build_nn", "tt_tree_pack", "tt_tree_from_blob", "tt_tree_upload",
    "tt_build_oct_device", "tt_build_oct_device_order", "tt_build_kd_device", "tt_build_vp_device", "tt_build_nn_device", "tt_tree_download",
    "tt_tree_copy_blob",
    "tt_sort_points", "tt_schedule_tiles", "tt_traverse_bh", "tt_traverse_pc", "tt_traverse_knn", "tt_traverse_vp", "tt_traverse_nn", "chase_records", "tt_diag_chase", "tt_diag_l2read",
    "build_info",
]


def _np_ptr(a: np.ndarray) -> int:
    return a.ctypes.data


def _stream_handle(stream) -> int:
    if stream is None:
        if not torch.cuda.is_available():
            return 0  # the library itself reports TT_ERR_CUDA: no CPU fallback
        stream = torch.cuda.current_stream()
    return int(stream.cuda_stream) if hasattr(stream, "cuda_stream") else int(stream)


def build_info() -> str:
    return L.load().tt_build_info().decode()


# --------------------------------------------------------------- host trees
class HostTree:
    """A canonical (preorder) tree built on the host by libtt's builders."""

    def __init__(self, handle: C.c_void_p, keepalive=None):
        self._h = handle
        self._keep = keepalive
        self.desc = L.tt_tree_desc()
        check(L.load().tt_host_tree_desc(self._h, C.byref(self.desc)), "tt_host_tree_desc")
        self.kind = {1: "oct", 2: "kd", 3: "vp", 4: "nn"}[self.desc.kind]
        self.dim = self.desc.dim
        self.height = self.desc.height
        self.n_nodes = self.desc.n_nodes
        self.n_points = self.desc.n_points

    def __del__(self):
        h = getattr(self, "_h", None)
        if h and L._lib is not None:
            L._lib.tt_host_tree_free(h)
            self._h = None

    def _arr(self, name: str, dtype, count: int) -> np.ndarray | None:
        ptr = getattr(self.desc, name)
        if not ptr:
            return None
        buf = (C.c_char * (count * np.dtype(dtype).itemsize)).from_address(ptr)
        return np.frombuffer(buf, dtype=dtype, count=count).copy()

    def array(self, name: str) -> np.ndarray | None:
        """Copy of one desc array (see tt_tree_desc in include/tt.h)."""
        n, d = self.n_nodes, self.dim
        spec = {
            "first_child": (np.int32, n), "skip": (np.int32, n), "level": (np.int32, n),
            "pbegin": (np.int32, n), "pcount": (np.int32, n), "split_dim": (np.int32, n),
            "split": (np.float32, n), "lo": (np.float32, n * d), "hi": (np.float32, n * d),
            "com": (np.float32, n * 4), "body": (np.int32, n), "in_child": (np.int32, n),
            "out_child": (np.int32, n), "r_in_max": (np.float32, n), "r_out_min": (np.float32, n),
            "tree_order": (np.int32, self.n_points),
        }[name]
        a = self._arr(name, *spec)
        if a is not None and name in ("lo", "hi"):
            a = a.reshape(n, d)
        if a is not None and name == "com":
            a = a.reshape(n, 4)
        return a

    @property
    def root_cube(self):
        return np.array(self.desc.root_center[:]), float(self.desc.root_side)

    def pack(self) -> np.ndarray:
        return tt_tree_pack(self)


def _host_points(pts: np.ndarray, width: int | None = None) -> np.ndarray:
    a = np.ascontiguousarray(np.asarray(pts, dtype=np.float32))
    if a.ndim != 2 or (width is not None and a.shape[1] != width):
        raise ValueError(f"expected a 2-D float32 array{'' if width is None else f' with {width} columns'}")
    return a


def build_kd(pts: np.ndarray, leaf_size: int = 1) -> HostTree:
    a = _host_points(pts)
    h = C.c_void_p()
    check(L.load().tt_build_kd(_np_ptr(a), a.shape[0], a.shape[1], a.shape[1], int(leaf_size), C.byref(h)),
          "tt_build_kd")
    return HostTree(h)


def build_oct(bodies: np.ndarray) -> HostTree:
    a = _host_points(bodies, 4)
    h = C.c_void_p()
    check(L.load().tt_build_oct(_np_ptr(a), a.shape[0], C.byref(h)), "tt_build_oct")
    return HostTree(h)


def build_vp(pts: np.ndarray) -> HostTree:
    a = _host_points(pts)
    h = C.c_void_p()
    check(L.load().tt_build_vp(_np_ptr(a), a.shape[0], a.shape[1], a.shape[1], C.byref(h)), "tt_build_vp")
    return HostTree(h)


def build_nn(pts: np.ndarray) -> HostTree:
    """NEXT-3: point-per-node kd-tree of the paper's NN benchmark (R21)."""
    a = _host_points(pts)
    h = C.c_void_p()
    check(L.load().tt_build_nn(_np_ptr(a), a.shape[0], a.shape[1], a.shape[1], C.byref(h)), "tt_build_nn")
    return HostTree(h)


def tt_tree_pack(host: HostTree) -> np.ndarray:
    """a0 on the host: the position-independent device blob (uint8 array)."""
    lib = L.load()
    n = C.c_size_t()
    check(lib.tt_tree_pack_size(C.byref(host.desc), C.byref(n)), "tt_tree_pack_size")
    blob = np.empty(n.value, dtype=np.uint8)
    check(lib.tt_tree_pack(C.byref(host.desc), _np_ptr(blob), n.value), "tt_tree_pack")
    return blob


# ------------------------------------------------------------- device trees
class Tree:
    """An uploaded tree (owns its device memory until freed / collected)."""

    def __init__(self, handle: C.c_void_p):
        self._h = handle
        info = L.tt_tree_info()
        check(L.load().tt_tree_get_info(self._h, C.byref(info)), "tt_tree_get_info")
        self.kind = {1: "oct", 2: "kd", 3: "vp", 4: "nn"}[info.kind]
        self.dim = info.dim
        self.height = info.height
        self.n_nodes = info.n_nodes
        self.n_points = info.n_points
        self.top_levels = info.top_levels
        self.top_count = info.top_count
        self.device_bytes = info.device_bytes
        self.device_blob = info.device_blob

    def free(self):
        h = getattr(self, "_h", None)
        if h and L._lib is not None:
            L._lib.tt_tree_free(h)
        self._h = None

    def __del__(self):
        self.free()


def tt_tree_upload(host: HostTree, stream=None) -> Tree:
    h = C.c_void_p()
    check(L.load().tt_tree_upload(C.byref(host.desc), C.c_void_p(_stream_handle(stream)), C.byref(h)),
          "tt_tree_upload")
    return Tree(h)


def tt_tree_from_blob(blob, stream=None) -> Tree:
    """Adopt a packed blob: numpy uint8 (host) or a CUDA uint8 tensor (device,
    e.g. after ``dist.broadcast``)."""
    h = C.c_void_p()
    if isinstance(blob, torch.Tensor):
        if not blob.is_cuda or blob.dtype != torch.uint8 or not blob.is_contiguous():
            raise ValueError("device blob must be a contiguous CUDA uint8 tensor")
        st = L.load().tt_tree_from_blob(C.c_void_p(blob.data_ptr()), blob.numel(), L.MEM_DEVICE,
                                        C.c_void_p(_stream_handle(stream)), C.byref(h))
    else:
        b = np.ascontiguousarray(blob, dtype=np.uint8)
        st = L.load().tt_tree_from_blob(_np_ptr(b), b.size, L.MEM_HOST, C.c_void_p(_stream_handle(stream)),
                                        C.byref(h))
    check(st, "tt_tree_from_blob")
    return Tree(h)


def tt_build_oct_device_order(bodies: torch.Tensor, order: torch.Tensor | None = None, stream=None):
    """tt_build_oct_device that also returns the bodies' tree order (leaf
    preorder; an int32 device tensor usable as a traversal `order`)."""
    _dev(bodies, torch.float32, "bodies", 4)
    if bodies.shape[1] != 4 or not bodies.is_contiguous():
        raise ValueError("bodies must be a contiguous (n, 4) float32 tensor")
    n = bodies.shape[0]
    if order is None:
        order = torch.empty(n, dtype=torch.int32, device=bodies.device)
    _dev(order, torch.int32, "order")
    if order.numel() < n or not order.is_contiguous():
        raise ValueError("order needs n contiguous int32 entries")
    h = C.c_void_p()
    check(L.load().tt_build_oct_device_order(bodies.data_ptr(), n, order.data_ptr(), C.c_void_p(_stream_handle(stream)),
                                             C.byref(h)), "tt_build_oct_device_order")
    return Tree(h), order


def tt_build_oct_device(bodies: torch.Tensor, stream=None) -> Tree:
    """NEXT-1: build the Barnes-Hut oct-tree on the GPU from (n, 4) device bodies."""
    _dev(bodies, torch.float32, "bodies", 4)
    if bodies.shape[1] != 4 or not bodies.is_contiguous():
        raise ValueError("bodies must be a contiguous (n, 4) float32 tensor")
    h = C.c_void_p()
    check(L.load().tt_build_oct_device(bodies.data_ptr(), bodies.shape[0], C.c_void_p(_stream_handle(stream)),
                                       C.byref(h)), "tt_build_oct_device")
    return Tree(h)


def tt_build_kd_device(pts: torch.Tensor, leaf_size: int = 1, stream=None) -> Tree:
    """NEXT-1: build the kd-tree on the GPU from (n, dim) device points."""
    _dev(pts, torch.float32, "pts", 1)
    h = C.c_void_p()
    check(L.load().tt_build_kd_device(pts.data_ptr(), pts.shape[0], pts.shape[1], pts.stride(0), int(leaf_size),
                                      C.c_void_p(_stream_handle(stream)), C.byref(h)), "tt_build_kd_device")
    return Tree(h)


def tt_build_nn_device(pts: torch.Tensor, stream=None) -> Tree:
    """Build the NN point-per-node kd-tree (R21) on the GPU from (n, dim) device points."""
    _dev(pts, torch.float32, "pts", 1)
    h = C.c_void_p()
    check(L.load().tt_build_nn_device(pts.data_ptr(), pts.shape[0], pts.shape[1], pts.stride(0),
                                      C.c_void_p(_stream_handle(stream)), C.byref(h)), "tt_build_nn_device")
    return Tree(h)


def tt_build_vp_device(pts: torch.Tensor, stream=None) -> Tree:
    """NEXT-1: build the vantage-point tree on the GPU from (n, dim) device points."""
    _dev(pts, torch.float32, "pts", 1)
    h = C.c_void_p()
    check(L.load().tt_build_vp_device(pts.data_ptr(), pts.shape[0], pts.shape[1], pts.stride(0),
                                      C.c_void_p(_stream_handle(stream)), C.byref(h)), "tt_build_vp_device")
    return Tree(h)


def tt_tree_copy_blob(tree: Tree, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """The packed device blob copied into a CUDA uint8 tensor (device to
    device, async on the stream): the send buffer of a tree broadcast."""
    if out is None:
        out = torch.empty(tree.device_bytes, dtype=torch.uint8, device="cuda")
    if not out.is_cuda or out.dtype != torch.uint8 or not out.is_contiguous():
        raise ValueError("out must be a contiguous CUDA uint8 tensor")
    check(L.load().tt_tree_copy_blob(tree._h, C.c_void_p(out.data_ptr()), out.numel(), L.MEM_DEVICE,
                                     C.c_void_p(_stream_handle(stream))), "tt_tree_copy_blob")
    return out


def tt_tree_download(tree: Tree) -> np.ndarray:
    """The packed device blob, copied to a host uint8 array."""
    out = np.empty(tree.device_bytes, dtype=np.uint8)
    check(L.load().tt_tree_download(tree._h, _np_ptr(out), out.size), "tt_tree_download")
    return out


# ------------------------------------------------------------------ launches
def _dev(t: torch.Tensor, dtype, name: str, cols: int | None = None) -> torch.Tensor:
    if not isinstance(t, torch.Tensor) or not t.is_cuda:
        raise TypeError(f"{name} must be a CUDA tensor (no CPU path exists)")
    if t.dtype != dtype:
        raise TypeError(f"{name} must be {dtype}, got {t.dtype}")
    if cols is not None and (t.dim() != 2 or t.shape[1] < cols or t.stride(1) != 1):
        raise ValueError(f"{name} must be 2-D with >= {cols} unit-stride columns")
    return t


@dataclass
class Stats:
    """Per-launch traversal counters (a6): see tt_stats in include/tt.h."""
    visits: torch.Tensor
    warp_fetches: torch.Tensor
    warp_steps: torch.Tensor
    warp_mode: torch.Tensor
    visit_hash: torch.Tensor | None = None   # int64 storage of the uint64 hashes
    visit_set: torch.Tensor | None = None
    point_tests: torch.Tensor | None = None

    @staticmethod
    def alloc(n: int, device, hashes: bool = False, point_tests: bool = False) -> "Stats":
        nw = (n + 31) // 32
        return Stats(torch.zeros(n, dtype=torch.int32, device=device),
                     torch.zeros(nw, dtype=torch.int32, device=device),
                     torch.zeros(nw, dtype=torch.int32, device=device),
                     torch.zeros(nw, dtype=torch.uint8, device=device),
                     torch.zeros(n, dtype=torch.int64, device=device) if hashes else None,
                     torch.zeros(n, dtype=torch.int64, device=device) if hashes else None,
                     torch.zeros(n, dtype=torch.int32, device=device) if point_tests else None)

    def hashes(self):
        """(visit_hash, visit_set) as numpy uint64 arrays."""
        return (self.visit_hash.cpu().numpy().view("uint64"), self.visit_set.cpu().numpy().view("uint64"))


def _lanes(order, n):
    """Launch lanes: one per entry of `order` (which indexes the point rows), else one per row."""
    return n if order is None else order.numel()


def _opts(mode, auto_min_depth, order, stats, n, variant="autoropes", switch_below=0):
    o = L.tt_traverse_opts()
    o.variant = L.VARIANT[variant]
    o.switch_below = int(switch_below)
    o.mode = L.MODE[mode] if isinstance(mode, str) else int(mode)
    o.auto_min_depth = -1 if auto_min_depth is None else int(auto_min_depth)
    keep = []
    if order is not None:
        _dev(order, torch.int32, "order")
        if order.dim() != 1 or not order.is_contiguous() or order.numel() > n:
            raise ValueError("order must be a contiguous 1-D index tensor over the point rows")
        o.order = order.data_ptr()
    if stats is not None:
        opt = lambda t: None if t is None else t.data_ptr()  # noqa: E731
        st = L.tt_stats(stats.visits.data_ptr(), stats.warp_fetches.data_ptr(), stats.warp_steps.data_ptr(),
                        stats.warp_mode.data_ptr(), opt(stats.visit_hash), opt(stats.visit_set),
                        opt(stats.point_tests))
        keep.append(st)
        o.stats = C.addressof(st)
    return o, keep


def tt_sort_points(tree: Tree, pts: torch.Tensor, out: torch.Tensor | None = None, keys: torch.Tensor | None = None,
                   stream=None) -> torch.Tensor:
    """a1: perm (int32 CUDA tensor; values are the uint32 permutation)."""
    _dev(pts, torch.float32, "pts", 3 if tree.kind == "oct" else tree.dim)
    n = pts.shape[0]
    if out is None:
        out = torch.empty(n, dtype=torch.int32, device=pts.device)
    kp = None
    if keys is not None:
        _dev(keys, torch.int64, "keys")
        kp = keys.data_ptr()
    check(L.load().tt_sort_points(tree._h, pts.data_ptr(), n, pts.stride(0), out.data_ptr(), kp,
                                  C.c_void_p(_stream_handle(stream))), "tt_sort_points")
    return out


def tt_schedule_tiles(tree: Tree, pts: torch.Tensor, perm: torch.Tensor, out: torch.Tensor | None = None,
                      stream=None) -> torch.Tensor:
    """a1b: `perm` with whole warp tiles reordered longest-estimated-first
    (include/tt.h).  out may be perm itself (in place)."""
    _dev(pts, torch.float32, "pts", 3 if tree.kind == "oct" else tree.dim)
    _dev(perm, torch.int32, "perm")
    n = perm.numel()
    if out is None:
        out = torch.empty_like(perm)
    _dev(out, torch.int32, "out")
    if out.numel() != n:
        raise ValueError("out must have perm's length")
    check(L.load().tt_schedule_tiles(tree._h, pts.data_ptr(), n, pts.stride(0), perm.data_ptr(), out.data_ptr(),
                                     C.c_void_p(_stream_handle(stream))), "tt_schedule_tiles")
    return out


def tt_traverse_bh(tree: Tree, bodies: torch.Tensor, theta: float, eps: float, out: torch.Tensor | None = None,
                   self_ids: torch.Tensor | None = None, order: torch.Tensor | None = None, mode="auto",
                   auto_min_depth: int | None = None, stats: Stats | None = None, stream=None,
                   variant: str = "autoropes") -> torch.Tensor:
    _dev(bodies, torch.float32, "bodies", 4)
    if bodies.shape[1] != 4 or not bodies.is_contiguous():
        raise ValueError("bodies must be a contiguous (n, 4) float32 tensor")
    n = bodies.shape[0]
    if out is None:
        out = torch.empty((n, 4), dtype=torch.float32, device=bodies.device)
    sp = None
    if self_ids is not None:
        _dev(self_ids, torch.int32, "self_ids")
        sp = self_ids.data_ptr()
    o, keep = _opts(mode, auto_min_depth, order, stats, n, variant)
    check(L.load().tt_traverse_bh(tree._h, bodies.data_ptr(), sp, _lanes(order, n), float(theta), float(eps), out.data_ptr(),
                                  C.byref(o), C.c_void_p(_stream_handle(stream))), "tt_traverse_bh")
    del keep
    return out


def tt_traverse_pc(tree: Tree, q: torch.Tensor, radius: float, out: torch.Tensor | None = None,
                   order: torch.Tensor | None = None, mode="auto", auto_min_depth: int | None = None,
                   stats: Stats | None = None, stream=None, variant: str = "autoropes") -> torch.Tensor:
    _dev(q, torch.float32, "q", tree.dim)
    n = q.shape[0]
    if out is None:
        out = torch.empty(n, dtype=torch.int32, device=q.device)
    o, keep = _opts(mode, auto_min_depth, order, stats, n, variant)
    check(L.load().tt_traverse_pc(tree._h, q.data_ptr(), _lanes(order, n), q.stride(0), float(radius), out.data_ptr(), C.byref(o),
                                  C.c_void_p(_stream_handle(stream))), "tt_traverse_pc")
    del keep
    return out


def tt_traverse_knn(tree: Tree, q: torch.Tensor, k: int, out_idx: torch.Tensor | None = None,
                    out_d2: torch.Tensor | None = None, order: torch.Tensor | None = None, mode="auto",
                    auto_min_depth: int | None = None, stats: Stats | None = None, stream=None,
                    variant: str = "autoropes", switch_below: int = 0):
    _dev(q, torch.float32, "q", tree.dim)
    n = q.shape[0]
    if out_idx is None:
        out_idx = torch.empty((n, k), dtype=torch.int32, device=q.device)
    if out_d2 is None:
        out_d2 = torch.empty((n, k), dtype=torch.float32, device=q.device)
    o, keep = _opts(mode, auto_min_depth, order, stats, n, variant, switch_below)
    check(L.load().tt_traverse_knn(tree._h, q.data_ptr(), _lanes(order, n), q.stride(0), int(k), out_idx.data_ptr(),
                                   out_d2.data_ptr(), C.byref(o), C.c_void_p(_stream_handle(stream))),
          "tt_traverse_knn")
    del keep
    return out_idx, out_d2


def tt_traverse_vp(tree: Tree, q: torch.Tensor, out_idx: torch.Tensor | None = None,
                   out_d2: torch.Tensor | None = None, order: torch.Tensor | None = None, mode="auto",
                   auto_min_depth: int | None = None, stats: Stats | None = None, stream=None,
                   variant: str = "autoropes"):
    _dev(q, torch.float32, "q", tree.dim)
    n = q.shape[0]
    if out_idx is None:
        out_idx = torch.empty(n, dtype=torch.int32, device=q.device)
    if out_d2 is None:
        out_d2 = torch.empty(n, dtype=torch.float32, device=q.device)
    o, keep = _opts(mode, auto_min_depth, order, stats, n, variant)
    check(L.load().tt_traverse_vp(tree._h, q.data_ptr(), _lanes(order, n), q.stride(0), out_idx.data_ptr(), out_d2.data_ptr(),
                                  C.byref(o), C.c_void_p(_stream_handle(stream))), "tt_traverse_vp")
    del keep
    return out_idx, out_d2


def tt_traverse_nn(tree: Tree, q: torch.Tensor, out_idx: torch.Tensor | None = None,
                   out_d2: torch.Tensor | None = None, order: torch.Tensor | None = None, mode="auto",
                   auto_min_depth: int | None = None, stats: Stats | None = None, stream=None):
    """NEXT-3: nearest neighbour over the point-per-node kd-tree (tt_build_nn)."""
    _dev(q, torch.float32, "q", tree.dim)
    n = q.shape[0]
    if out_idx is None:
        out_idx = torch.empty(n, dtype=torch.int32, device=q.device)
    if out_d2 is None:
        out_d2 = torch.empty(n, dtype=torch.float32, device=q.device)
    o, keep = _opts(mode, auto_min_depth, order, stats, n, "autoropes")
    check(L.load().tt_traverse_nn(tree._h, q.data_ptr(), _lanes(order, n), q.stride(0), out_idx.data_ptr(),
                                  out_d2.data_ptr(), C.byref(o), C.c_void_p(_stream_handle(stream))), "tt_traverse_nn")
    del keep
    return out_idx, out_d2


# ---------------------------------------------------------------- diagnostics
def chase_records(nrec: int, device, seed: int = 0) -> torch.Tensor:
    """nrec 32-B records forming one random cycle (int32 at word 4 = next
    index), for tt_diag_chase.  Plumbing only (a permutation)."""
    g = torch.Generator(device=device).manual_seed(seed)
    perm = torch.randperm(nrec, device=device, generator=g, dtype=torch.int64)
    rec = torch.zeros((nrec, 8), dtype=torch.int32, device=device)
    rec[perm, 4] = torch.roll(perm, -1).to(torch.int32)
    rec[:, 5] = 1
    return rec


def tt_diag_chase(records: torch.Tensor, steps: int, per_lane: bool = False, ctas_per_sm: int = 0,
                  stream=None) -> None:
    """Dependent 32-B record chase with the traversal kernels' launch shape
    (the walk's latency ceiling; include/tt.h).  Asynchronous; time it."""
    _dev(records, torch.int32, "records", 8)
    sink = torch.zeros(1, dtype=torch.int32, device=records.device)
    check(L.load().tt_diag_chase(records.data_ptr(), records.shape[0], int(bool(per_lane)), int(steps),
                                 int(ctas_per_sm), sink.data_ptr(), C.c_void_p(_stream_handle(stream))),
          "tt_diag_chase")


def tt_diag_l2read(buf: torch.Tensor, reps: int, stream=None) -> None:
    """L2-resident streaming read of `buf` (the L2 read-bandwidth ceiling;
    include/tt.h).  Asynchronous; time it."""
    if not buf.is_cuda or not buf.is_contiguous():
        raise ValueError("buf must be a contiguous CUDA tensor")
    sink = torch.zeros(1, dtype=torch.int32, device=buf.device)
    nbytes = buf.numel() * buf.element_size() // 32 * 32
    check(L.load().tt_diag_l2read(buf.data_ptr(), nbytes, int(reps), sink.data_ptr(),
                                  C.c_void_p(_stream_handle(stream))), "tt_diag_l2read")

"""Brute-force definitions in numpy, used to pin the oracle (tests only).

These are the plain definitions of what each traversal computes (no tree):
  * pinned fp32 squared distance, R0: per-dimension float32
    subtract, square, sequential add -- written with explicit float32 numpy
    ops in dimension order (NOT np.sum, which is pairwise);
  * PC count  = #{j : d2(q, p_j) <= rn(r*r)}            (R1)
  * kNN       = k smallest (d2, j) lexicographically      (R4)
  * VP / NN   = argmin (d2, j)
  * BH theta=0: direct O(n^2) sum of m_j (x_j - x_i)/(|x_j - x_i|^2+eps^2)^{3/2}
    over j != i, in fp64 (textbook softened gravity, G=1, R7).
"""
from __future__ import annotations

import numpy as np


def pinned_d2(q: np.ndarray, p: np.ndarray) -> np.ndarray:
    """(m, D) x (n, D) -> (m, n) float32 pinned squared distances."""
    q = np.asarray(q, np.float32)
    p = np.asarray(p, np.float32)
    t = (q[:, None, 0] - p[None, :, 0]).astype(np.float32)
    s = (t * t).astype(np.float32)
    for d in range(1, q.shape[1]):
        t = (q[:, None, d] - p[None, :, d]).astype(np.float32)
        s = (s + (t * t).astype(np.float32)).astype(np.float32)
    return s


def pc_counts(q, p, radius) -> np.ndarray:
    r2 = np.float32(np.float32(radius) * np.float32(radius))
    out = np.zeros(len(q), np.uint32)
    for s in range(0, len(q), 512):
        out[s:s + 512] = (pinned_d2(q[s:s + 512], p) <= r2).sum(axis=1)
    return out


def knn(q, p, k):
    m, n = len(q), len(p)
    idx = np.full((m, k), -1, np.int64)
    d2 = np.full((m, k), np.inf, np.float32)
    for s in range(0, m, 512):
        D = pinned_d2(q[s:s + 512], p)
        for i in range(D.shape[0]):
            order = np.lexsort((np.arange(n), D[i]))[:k]
            idx[s + i, :len(order)] = order
            d2[s + i, :len(order)] = D[i, order]
    return idx, d2


def nn(q, p):
    idx, d2 = knn(q, p, 1)
    return idx[:, 0], d2[:, 0]


def direct_sum(bodies: np.ndarray, eps: float) -> np.ndarray:
    b = np.asarray(bodies, np.float64)
    x, m = b[:, :3], b[:, 3]
    e2 = float(np.float32(eps)) ** 2
    acc = np.zeros((len(b), 3))
    for s in range(0, len(b), 256):
        dx = x[None, :, :] - x[s:s + 256, None, :]
        r2 = (dx * dx).sum(-1) + e2
        inv3 = r2 ** -1.5
        for i in range(dx.shape[0]):
            inv3[i, s + i] = 0.0  # j != i
        acc[s:s + 256] = (m[None, :, None] * dx * inv3[..., None]).sum(1)
    return acc


def morton63(x: np.ndarray, center: np.ndarray, side: float) -> np.ndarray:
    """Octant-path code of each point through the cube hierarchy, by integer
    quantisation floor((x - lo) / side * 2^21) (an independent formulation of
    the repeated centre comparisons; exact when the quotient is exact)."""
    lo = center - side / 2.0
    q = np.floor((np.asarray(x, np.float64)[:, :3] - lo) / side * (1 << 21)).astype(np.int64)
    q = np.clip(q, 0, (1 << 21) - 1).astype(np.uint64)
    code = np.zeros(len(x), np.uint64)
    for lvl in range(20, -1, -1):
        o = ((q[:, 0] >> np.uint64(lvl)) & np.uint64(1)) | \
            (((q[:, 1] >> np.uint64(lvl)) & np.uint64(1)) << np.uint64(1)) | \
            (((q[:, 2] >> np.uint64(lvl)) & np.uint64(1)) << np.uint64(2))
        code = (code << np.uint64(3)) | o
    return code

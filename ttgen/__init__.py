"""Seeded synthetic input generators shared by the oracle tests and the CUDA path.

This module holds NO arithmetic of the traversal method (no distances, no
trees, no opening tests): it only draws the point sets the paper's workloads
are shaped like, so that both sides of every parity test read the same bytes.

Workload shapes (§6.1.2; recipe in DESIGN.md §3):
  * ``uniform``   - uniform [0,1)^D points (PC "Random" input).
  * ``plummer``   - Plummer-model bodies of equal mass (BH "Plummer" input,
                    "1 million bodies of equal mass generated from the Plummer
                    model"), Aarseth-Henon-Wielen sampling.
  * ``gaussian_mixture`` - clustered D-dim points (stand-in for the paper's
                    random-projection inputs Covtype/Mnist).
  * ``permutation`` - the seeded shuffle used for "unsorted" inputs
                    (P:L1116-1117).

RNG: numpy PCG64 (``np.random.default_rng(seed)``), computed in float64 and
rounded once to float32.
"""
from __future__ import annotations

import numpy as np

__all__ = ["uniform", "plummer", "plummer_velocities", "gaussian_mixture", "permutation", "CONFIGS"]


def uniform(n: int, dim: int, seed: int) -> np.ndarray:
    """(n, dim) float32, iid U[0,1)."""
    rng = np.random.default_rng(seed)
    return rng.random((n, dim), dtype=np.float64).astype(np.float32)


def plummer(n: int, seed: int) -> np.ndarray:
    """(n, 4) float32 rows (x, y, z, m): Plummer sphere, equal masses 1/n.

    Aarseth, Henon & Wielen (1974): r = (X^{-2/3} - 1)^{-1/2} with
    X ~ U(0, 0.999] (truncates the unbounded tail), isotropic direction,
    positions scaled by 3*pi/16 (standard N-body units).
    """
    rng = np.random.default_rng(seed)
    x1 = rng.random(n) * 0.999
    x1 = np.where(x1 <= 0.0, 1e-300, x1)  # (0, 0.999]
    r = 1.0 / np.sqrt(x1 ** (-2.0 / 3.0) - 1.0)
    cost = rng.random(n) * 2.0 - 1.0
    phi = rng.random(n) * (2.0 * np.pi)
    sint = np.sqrt(np.maximum(0.0, 1.0 - cost * cost))
    scale = 3.0 * np.pi / 16.0
    out = np.empty((n, 4), dtype=np.float64)
    out[:, 0] = scale * r * sint * np.cos(phi)
    out[:, 1] = scale * r * sint * np.sin(phi)
    out[:, 2] = scale * r * cost
    out[:, 3] = 1.0 / max(n, 1)
    return out.astype(np.float32)


def plummer_velocities(bodies: np.ndarray, seed: int) -> np.ndarray:
    """(n, 4) float32 rows (vx, vy, vz, 0) for `plummer` bodies: Aarseth,
    Henon & Wielen (1974) von Neumann rejection for q = v / v_esc with
    g(q) ~ q^2 (1 - q^2)^{7/2}, v_esc = sqrt(2) (1 + r^2)^{-1/4}, isotropic
    direction, in the same standard units as the positions (velocities scaled
    by sqrt(16 / (3 pi))).  Separate RNG stream: positions are unchanged."""
    rng = np.random.default_rng(seed)
    n = len(bodies)
    pscale = 3.0 * np.pi / 16.0
    r = np.linalg.norm(np.asarray(bodies, np.float64)[:, :3], axis=1) / pscale
    q = np.empty(n)
    todo = np.arange(n)
    while len(todo):
        x = rng.random(len(todo))
        y = rng.random(len(todo)) * 0.1
        ok = y < x * x * (1.0 - x * x) ** 3.5
        q[todo[ok]] = x[ok]
        todo = todo[~ok]
    v = q * np.sqrt(2.0) * (1.0 + r * r) ** -0.25 * np.sqrt(16.0 / (3.0 * np.pi))
    cost = rng.random(n) * 2.0 - 1.0
    phi = rng.random(n) * (2.0 * np.pi)
    sint = np.sqrt(np.maximum(0.0, 1.0 - cost * cost))
    out = np.zeros((n, 4))
    out[:, 0] = v * sint * np.cos(phi)
    out[:, 1] = v * sint * np.sin(phi)
    out[:, 2] = v * cost
    return out.astype(np.float32)


def gaussian_mixture(n: int, dim: int, seed: int, components: int = 32,
                     sigma: float = 0.05) -> np.ndarray:
    """(n, dim) float32: equal-weight isotropic Gaussian mixture.

    Component means ~ U[0,1)^dim, standard deviation ``sigma`` per axis.
    """
    rng = np.random.default_rng(seed)
    means = rng.random((components, dim))
    comp = rng.integers(0, components, size=n)
    pts = means[comp] + sigma * rng.standard_normal((n, dim))
    return pts.astype(np.float32)


def permutation(n: int, seed: int) -> np.ndarray:
    """Seeded random permutation of range(n) (int64)."""
    return np.random.default_rng(seed).permutation(n)


# The BASELINE.json configs as generator recipes.
CONFIGS = {
    "pc_10k_3d": dict(kind="pc", n=10_000, dim=3, seed=1, radius=0.1, leaf=1),
    "bh_1m_plummer": dict(kind="bh", n=1_000_000, seed=2, theta=0.5, eps=0.05),
    "knn_1m_7d": dict(kind="knn", n=1_000_000, m=1_000_000, dim=7, seed=3,
                      qseed=4, k=8, leaf=8),
    "vp_1m_16d": dict(kind="vp", n=1_000_000, m=1_000_000, dim=16, seed=5,
                      qseed=6, perm_seed=7),
    "bh_16m_plummer": dict(kind="bh", n=16_777_216, seed=8, theta=0.5, eps=0.05),
    "knn_16m_7d": dict(kind="knn", n=16_777_216, m=16_777_216, dim=7, seed=9,
                       qseed=10, k=8, leaf=8),
}

"""SU3Bench-style lattice inputs (config 3).

Layout: complex128 A[sites][4][3][3] (one SU(3) link matrix per site and
direction), B[4][3][3], stored as float64 (..., 2) = (re, im) interleaved, i.e.
exactly numpy's complex128 memory layout.

Two recipes (PAPER.md:933-944 names the
kernel only):
* ``constant``: A = 1 + 0i, B = 1/3 + 0i everywhere (SU3Bench's own
  initialisation style).
* ``random``: Haar-like random SU(3) matrices built from two uniform complex
  vectors (Gram-Schmidt, third row = conj cross product => det = 1), seeded.
"""
import numpy as np

from .stream import uniform

SEED_SU3 = 2022


def lattice_sites(L):
    return L ** 4


def _random_su3(n, seed, skip=0):
    u = uniform(seed, n * 12, skip=skip * 12).reshape(n, 2, 3, 2) * 2.0 - 1.0
    v1 = u[:, 0, :, 0] + 1j * u[:, 0, :, 1]
    v2 = u[:, 1, :, 0] + 1j * u[:, 1, :, 1]
    v1 = v1 / np.linalg.norm(v1, axis=1, keepdims=True)
    v2 = v2 - np.sum(np.conj(v1) * v2, axis=1, keepdims=True) * v1
    v2 = v2 / np.linalg.norm(v2, axis=1, keepdims=True)
    v3 = np.conj(np.cross(v1, v2))
    return np.stack([v1, v2, v3], axis=1)          # rows are orthonormal


def make_lattice(sites, kind="random", seed=SEED_SU3, first_site=0):
    """Return (A, B) as complex128 arrays [sites,4,3,3] and [4,3,3]: sites
    [first_site, first_site + sites) of the global lattice (a rank's shard;
    B is replicated)."""
    if kind == "constant":
        A = np.ones((sites, 4, 3, 3), dtype=np.complex128)
        B = np.full((4, 3, 3), 1.0 / 3.0, dtype=np.complex128)
        return A, B
    if kind != "random":
        raise ValueError(kind)
    A = _random_su3(sites * 4, seed, skip=first_site * 4).reshape(sites, 4, 3, 3)
    B = _random_su3(4, seed + 1).reshape(4, 3, 3)
    return np.ascontiguousarray(A), np.ascontiguousarray(B)

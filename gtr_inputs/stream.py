"""Vectorised uniform draws for table generation.

The tables are filled from the 63-bit LCG stream the XSBench/RSBench proxy apps
use for their data ([ext]: s <- (a*s + c) mod 2^63, a = 2806196910506780709,
c = 1, U = s / 2^63).  Here it is only a data source: state k of the stream is
produced by affine jump-ahead in numpy so 10^8 draws take about a second.  The
lookup kernels' own sampling is NOT taken from here -- the
oracle and the CUDA path each implement it on their own.
"""
import numpy as np

A = 2806196910506780709
C = 1
MASK63 = (1 << 63) - 1


def _jump(n):
    """(a_n, c_n) with s_{k+n} = a_n * s_k + c_n (mod 2^63), python ints."""
    a_n, c_n = 1, 0
    a, c = A, C
    while n:
        if n & 1:
            a_n = (a_n * a) & MASK63
            c_n = (c_n * a + c) & MASK63
        c = (c * (a + 1)) & MASK63
        a = (a * a) & MASK63
        n >>= 1
    return a_n, c_n


def lcg_states(seed, n):
    """States s_1..s_n of the stream started at `seed` (uint64 array)."""
    out = np.empty(n, dtype=np.uint64)
    if n == 0:
        return out
    out[0] = (A * seed + C) & MASK63
    filled = 1
    mask = np.uint64(MASK63)
    with np.errstate(over="ignore"):
        while filled < n:
            take = min(filled, n - filled)
            a_f, c_f = _jump(filled)
            # uint64 products wrap mod 2^64; masking reduces mod 2^63 exactly.
            out[filled:filled + take] = (out[:take] * np.uint64(a_f) + np.uint64(c_f)) & mask
            filled += take
    return out


def uniform(seed, n, skip=0):
    """n draws U = s / 2^63 in [0, 1) (u64 -> f64 rounds to nearest, /2^63 exact),
    starting after the first `skip` draws of the stream (shards of a global
    input)."""
    if skip:
        a_s, c_s = _jump(skip)
        seed = (a_s * seed + c_s) & MASK63
    return lcg_states(seed, n).astype(np.float64) / float(1 << 63)

"""ctypes loader for the C oracle (liboracle.so).

TEST INFRASTRUCTURE ONLY: importable from tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference legs.  The product package
(paper_conf_cgo_hubercgtddcd22_b200) never imports this module.
"""
import ctypes as C
import os
import subprocess

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SOURCES = ["xs.c", "su3.c", "rs.c", "forkjoin.c", "semantics.c"]
LIB = os.path.join(HERE, "liboracle.so")
CFLAGS = ["-O2", "-std=c11", "-D_GNU_SOURCE", "-ffp-contract=off", "-fno-fast-math",
          "-fPIC", "-shared", "-Wall", "-Wextra", "-Wno-unused-parameter"]


def build(force=False):
    srcs = [os.path.join(HERE, s) for s in SOURCES] + [os.path.join(HERE, "oracle.h")]
    if not force and os.path.exists(LIB):
        lt = os.path.getmtime(LIB)
        if all(os.path.getmtime(s) <= lt for s in srcs):
            return LIB
    cmd = ["gcc"] + CFLAGS + [os.path.join(HERE, s) for s in SOURCES] + ["-o", LIB + ".tmp", "-lm", "-lpthread"]
    subprocess.check_call(cmd)
    os.replace(LIB + ".tmp", LIB)
    return LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(LIB)
        u64, i64, i32, dbl, vp = C.c_uint64, C.c_int64, C.c_int32, C.c_double, C.c_void_p
        L.orc_lcg_next.restype = u64; L.orc_lcg_next.argtypes = [u64]
        L.orc_lcg_double.restype = dbl; L.orc_lcg_double.argtypes = [C.POINTER(u64)]
        L.orc_lcg_ff.restype = u64; L.orc_lcg_ff.argtypes = [u64, u64]
        L.orc_pick_mat.restype = C.c_int; L.orc_pick_mat.argtypes = [C.POINTER(u64)]
        L.orc_xs_build_egrid.restype = None; L.orc_xs_build_egrid.argtypes = [vp, i64, i64, vp]
        L.orc_xs_build_index_grid.restype = None
        L.orc_xs_build_index_grid.argtypes = [vp, i64, i64, vp, i64, vp]
        L.orc_grid_search.restype = i64; L.orc_grid_search.argtypes = [i64, vp, dbl]
        L.orc_nuclide_search.restype = i64; L.orc_nuclide_search.argtypes = [vp, dbl, i64, i64]
        L.orc_xs_build_hash_grid.restype = None
        L.orc_xs_build_hash_grid.argtypes = [vp, i64, i64, i32, vp]
        L.orc_xs_lookup.restype = None
        L.orc_xs_lookup.argtypes = [vp, u64, u64, vp, vp, vp, vp]
        L.orc_xs_run.restype = None
        L.orc_xs_run.argtypes = [vp, u64, u64, u64, C.c_int, vp, vp, vp, vp, vp]
        L.orc_su3_mat_nn.restype = None; L.orc_su3_mat_nn.argtypes = [i64, vp, vp, vp, C.c_int]
        L.orc_fast_exp.restype = dbl; L.orc_fast_exp.argtypes = [dbl]
        L.orc_fast_nuclear_W.restype = Cplx; L.orc_fast_nuclear_W.argtypes = [Cplx]
        L.orc_rs_faddeeva_constants.restype = None
        L.orc_rs_faddeeva_constants.argtypes = [vp, vp, vp, vp]
        L.orc_rs_lookup.restype = None; L.orc_rs_lookup.argtypes = [vp, u64, u64, vp, vp, vp]
        L.orc_rs_run.restype = None
        L.orc_rs_run.argtypes = [vp, u64, u64, u64, C.c_int, vp, vp, vp, vp, vp]
        L.orc_rs_work.restype = None; L.orc_rs_work.argtypes = [vp, u64, u64, u64, C.c_int, vp]
        L.orc_rs_flops.restype = dbl; L.orc_rs_flops.argtypes = [vp, C.POINTER(dbl)]
        L.orc_fj_team.restype = u64; L.orc_fj_team.argtypes = [i32, i32, i64, i32, i32]
        L.orc_fj_host_team.restype = u64
        L.orc_fj_host_team.argtypes = [i32, i64, i32, i32, C.POINTER(dbl)]
        L.orc_sem_expected.restype = C.c_int
        L.orc_sem_expected.argtypes = [i32, i32, i32, vp, i64]
        _lib = L
    return _lib


class Cplx(C.Structure):
    _fields_ = [("r", C.c_double), ("i", C.c_double)]


class XsTables(C.Structure):
    _fields_ = [("n_iso", C.c_int64), ("n_gp", C.c_int64), ("n_union", C.c_int64),
                ("max_num_nucs", C.c_int32),
                ("grid", C.c_void_p), ("egrid", C.c_void_p), ("index_grid", C.c_void_p),
                ("num_nucs", C.c_void_p), ("mats", C.c_void_p), ("concs", C.c_void_p),
                ("grid_type", C.c_int32), ("hash_bins", C.c_int32), ("hash_index", C.c_void_p)]


class RsTables(C.Structure):
    _fields_ = [("n_nuc", C.c_int64), ("max_poles", C.c_int64), ("max_windows", C.c_int64),
                ("max_num_nucs", C.c_int32),
                ("n_windows", C.c_void_p), ("poles", C.c_void_p), ("windows", C.c_void_p),
                ("k0rs", C.c_void_p), ("num_nucs", C.c_void_p), ("mats", C.c_void_p),
                ("concs", C.c_void_p)]


def _p(a):
    return a.ctypes.data_as(C.c_void_p)


# ---------------------------------------------------------------- sampling
def lcg_next(s):
    return lib().orc_lcg_next(s)


def lcg_ff(seed, n):
    return lib().orc_lcg_ff(seed, n)


def lcg_double(seed):
    s = C.c_uint64(seed)
    d = lib().orc_lcg_double(C.byref(s))
    return d, s.value


def pick_mat(seed):
    s = C.c_uint64(seed)
    m = lib().orc_pick_mat(C.byref(s))
    return m, s.value


def grid_search(a, q):
    a = np.ascontiguousarray(a, dtype=np.float64)
    return lib().orc_grid_search(len(a), _p(a), q)


def nuclide_search(grid_n, q, low, high):
    g = np.ascontiguousarray(grid_n, dtype=np.float64)
    return lib().orc_nuclide_search(_p(g), q, low, high)


# ---------------------------------------------------------------- XS
class XsProblem:
    """Oracle-side tables: the generator's grid + the oracle's own unionized
    energy grid and index grid."""

    def __init__(self, t, build_index=True, grid_type=0, hash_bins=10000):
        self.src = t
        self.grid = np.ascontiguousarray(t["grid"], dtype=np.float64)
        self.n_iso, self.n_gp = int(t["n_iso"]), int(t["n_gp"])
        self.n_union = self.n_iso * self.n_gp
        self.num_nucs = np.ascontiguousarray(t["num_nucs"], dtype=np.int32)
        self.mats = np.ascontiguousarray(t["mats"], dtype=np.int32)
        self.concs = np.ascontiguousarray(t["concs"], dtype=np.float64)
        self.egrid = np.empty(self.n_union, dtype=np.float64)
        lib().orc_xs_build_egrid(_p(self.grid), self.n_iso, self.n_gp, _p(self.egrid))
        self.index_grid = None
        if build_index:
            self.index_grid = np.empty((self.n_union, self.n_iso), dtype=np.int32)
            lib().orc_xs_build_index_grid(_p(self.grid), self.n_iso, self.n_gp, _p(self.egrid),
                                          self.n_union, _p(self.index_grid))
        self.grid_type, self.hash_bins, self.hash_index = grid_type, hash_bins, None
        if grid_type == 2:
            self.hash_index = np.empty((hash_bins, self.n_iso), dtype=np.int32)
            lib().orc_xs_build_hash_grid(_p(self.grid), self.n_iso, self.n_gp, hash_bins, _p(self.hash_index))
        self.ct = XsTables(self.n_iso, self.n_gp, self.n_union, self.mats.shape[1],
                           _p(self.grid).value, _p(self.egrid).value,
                           _p(self.index_grid).value if self.index_grid is not None else None,
                           _p(self.num_nucs).value, _p(self.mats).value, _p(self.concs).value,
                           grid_type, hash_bins,
                           _p(self.hash_index).value if self.hash_index is not None else None)

    def lookup(self, i, seed):
        mat, am = C.c_int32(), C.c_int32()
        u = C.c_int64()
        macro = np.zeros(5, dtype=np.float64)
        lib().orc_xs_lookup(C.byref(self.ct), i, seed, C.byref(mat), C.byref(u), _p(macro), C.byref(am))
        return mat.value, u.value, macro, am.value

    def run(self, first, n, seed, nthreads=1, verify=False):
        out = np.zeros(18, dtype=np.uint64)
        v = None
        if verify:
            v = {"mat": np.zeros(n, np.uint8), "u": np.zeros(n, np.uint32),
                 "am": np.zeros(n, np.uint8), "macro": np.zeros((n, 5), np.float64)}
            lib().orc_xs_run(C.byref(self.ct), first, n, seed, nthreads, _p(out),
                             _p(v["mat"]), _p(v["u"]), _p(v["am"]), _p(v["macro"]))
        else:
            lib().orc_xs_run(C.byref(self.ct), first, n, seed, nthreads, _p(out),
                             None, None, None, None)
        return out, v


# ---------------------------------------------------------------- SU3
def su3_mat_nn(A, B, nthreads=1):
    A = np.ascontiguousarray(A, dtype=np.complex128)
    B = np.ascontiguousarray(B, dtype=np.complex128)
    Cm = np.empty_like(A)
    lib().orc_su3_mat_nn(A.shape[0], _p(A), _p(B), _p(Cm), nthreads)
    return Cm


# ---------------------------------------------------------------- RS
def fast_nuclear_W(z):
    r = lib().orc_fast_nuclear_W(Cplx(z.real, z.imag))
    return complex(r.r, r.i)


def fast_exp(x):
    return lib().orc_fast_exp(x)


def rs_faddeeva_constants():
    """(an[10], denominator_left[10], prefactor, (a, b, c, d)) as orc_fast_nuclear_W uses them."""
    an, dl, asym = np.zeros(10), np.zeros(10), np.zeros(4)
    pre = C.c_double()
    lib().orc_rs_faddeeva_constants(_p(an), _p(dl), C.byref(pre), _p(asym))
    return an, dl, pre.value, asym


class RsProblem:
    def __init__(self, t):
        self.src = t
        self.n_windows = np.ascontiguousarray(t["n_windows"], dtype=np.int32)
        self.poles = np.ascontiguousarray(t["poles"])
        self.windows = np.ascontiguousarray(t["windows"])
        self.k0rs = np.ascontiguousarray(t["k0rs"], dtype=np.float64)
        self.num_nucs = np.ascontiguousarray(t["num_nucs"], dtype=np.int32)
        self.mats = np.ascontiguousarray(t["mats"], dtype=np.int32)
        self.concs = np.ascontiguousarray(t["concs"], dtype=np.float64)
        self.ct = RsTables(int(t["n_nuc"]), int(t["max_poles"]), int(t["max_windows"]),
                           self.mats.shape[1], _p(self.n_windows).value, _p(self.poles).value,
                           _p(self.windows).value, _p(self.k0rs).value, _p(self.num_nucs).value,
                           _p(self.mats).value, _p(self.concs).value)

    def lookup(self, i, seed):
        mat, am = C.c_int32(), C.c_int32()
        macro = np.zeros(4, dtype=np.float64)
        lib().orc_rs_lookup(C.byref(self.ct), i, seed, C.byref(mat), _p(macro), C.byref(am))
        return mat.value, macro, am.value

    def run(self, first, n, seed, nthreads=1, verify=False):
        out = np.zeros(18, dtype=np.uint64)
        margin = C.c_double()
        v = None
        if verify:
            v = {"mat": np.zeros(n, np.uint8), "am": np.zeros(n, np.uint8),
                 "macro": np.zeros((n, 4), np.float64)}
            lib().orc_rs_run(C.byref(self.ct), first, n, seed, nthreads, _p(out),
                             _p(v["mat"]), _p(v["am"]), _p(v["macro"]), C.byref(margin))
        else:
            lib().orc_rs_run(C.byref(self.ct), first, n, seed, nthreads, _p(out),
                             None, None, None, C.byref(margin))
        return out, v, margin.value

    def work(self, first, n, seed, nthreads=1):
        """Algorithmic fp64 work of lookups [first, first+n): (counts, flops,
        transcendentals); counts = (nuclide visits, Abrarov poles, asymptotic
        poles).  Weights in oracle/rs.c."""
        counts = np.zeros(3, dtype=np.uint64)
        lib().orc_rs_work(C.byref(self.ct), first, n, seed, nthreads, _p(counts))
        tr = C.c_double()
        fl = lib().orc_rs_flops(_p(counts), C.byref(tr))
        return counts, fl, tr.value


# ---------------------------------------------------------------- fork/join
def fj_team(g, T, R, body, K=1):
    return lib().orc_fj_team(g, T, R, body, K)


def fj_host_team(T, R, body, K=1):
    ns = C.c_double()
    r = lib().orc_fj_host_team(T, R, body, K, C.byref(ns))
    return r, ns.value


def sem_expected(test_id, G, T):
    out = np.zeros(10 * G * T + 21 * G + 16, dtype=np.uint64)
    n = lib().orc_sem_expected(test_id, G, T, _p(out), len(out))
    if n < 0:
        raise ValueError("bad semantics test id")
    return out[:n].copy()

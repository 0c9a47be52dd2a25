"""Thin ctypes binding of libgtr.so -- the C ABI in include/gtr.h.

Argument marshalling only: every function has the C name, takes device
pointers as ints or torch tensors, `stream` as a torch.cuda.Stream, an int
handle or None (= torch's current stream), and raises GtrError on a non-zero
status.  No computation happens here, and there is no fallback: if the CUDA
library is missing the import of this module fails loudly.
"""
import ctypes as C
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("GTR_LIB", os.path.join(_HERE, "libgtr.so"))   # GTR_LIB: experiments

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing -- build it with "
                      "`python -m paper_conf_cgo_hubercgtddcd22_b200.build` (no CPU fallback exists)")
_lib = C.CDLL(LIB_PATH)

# ---------------------------------------------------------------- constants
GTR_OK, GTR_EINVAL, GTR_ECUDA, GTR_ENOMEM, GTR_EHEAP, GTR_EDEVICE, GTR_EUNSUPPORTED = 0, -1, -2, -3, -4, -5, -6
GENERIC, GENERIC_CASCADE, CSM, SPMD, NATIVE = 0, 1, 2, 3, 4
PL_RUNTIME, PL_GLOBAL, PL_SHARED_STATIC, PL_STACK, PL_COALESCED = 0, 1, 2, 3, 4
F_BCAST_1BAR, F_SEPARATE_GUARDS, F_PLAIN, F_HISTORY, F_TMA, F_NATIVE_BUCKETED, F_SORTED = 1, 2, 4, 8, 16, 32, 64
K_XS, K_SU3, K_RS, K_FORKJOIN, K_SEMANTICS, K_BARRIER_FLOOR = 0, 1, 2, 3, 4, 5
MODE_NAMES = {GENERIC: "generic", GENERIC_CASCADE: "cascade", CSM: "csm", SPMD: "spmd", NATIVE: "native"}
PL_NAMES = {PL_RUNTIME: "runtime", PL_GLOBAL: "global", PL_SHARED_STATIC: "shared_static", PL_STACK: "stack",
            PL_COALESCED: "coalesced"}


class GtrError(RuntimeError):
    def __init__(self, fn, status):
        super().__init__(f"{fn}: {gtr_strerror(status)} ({status})")
        self.status = status


# ---------------------------------------------------------------- structs
class gtr_launch_cfg(C.Structure):
    _fields_ = [("num_teams", C.c_int32), ("thread_limit", C.c_int32), ("mode", C.c_int32),
                ("placement", C.c_int32), ("fold", C.c_int32), ("smem_stack_bytes", C.c_uint32),
                ("flags", C.c_int32)]


class gtr_variant_info(C.Structure):
    _fields_ = [("regs", C.c_int32), ("static_smem", C.c_int32), ("dyn_smem", C.c_int32),
                ("local_bytes", C.c_int32), ("block_threads", C.c_int32),
                ("teams_per_sm", C.c_int32), ("num_teams", C.c_int32)]


class gtr_xs_tables(C.Structure):
    _fields_ = [("n_iso", C.c_int64), ("n_gp", C.c_int64), ("n_union", C.c_int64),
                ("max_num_nucs", C.c_int32), ("egrid", C.c_void_p), ("index_grid", C.c_void_p),
                ("grid", C.c_void_p), ("num_nucs", C.c_void_p), ("mats", C.c_void_p),
                ("concs", C.c_void_p), ("grid_type", C.c_int32), ("hash_bins", C.c_int32),
                ("hash_index", C.c_void_p), ("energies", C.c_void_p),
                ("union_bins", C.c_void_p), ("union_bins_log2", C.c_int32)]


XS_UNIONIZED, XS_NUCLIDE, XS_HASH = 0, 1, 2


class gtr_xs_verify(C.Structure):
    _fields_ = [("mat", C.c_void_p), ("u", C.c_void_p), ("am", C.c_void_p), ("macro", C.c_void_p)]


class gtr_xs_request(C.Structure):
    _fields_ = [("first", C.c_uint64), ("n", C.c_uint64), ("seed", C.c_uint64)]


class gtr_rs_tables(C.Structure):
    _fields_ = [("n_nuc", C.c_int64), ("max_poles", C.c_int64), ("max_windows", C.c_int64),
                ("max_num_nucs", C.c_int32), ("n_windows", C.c_void_p), ("poles", C.c_void_p),
                ("windows", C.c_void_p), ("k0rs", C.c_void_p), ("num_nucs", C.c_void_p),
                ("mats", C.c_void_p), ("concs", C.c_void_p), ("poles_wide", C.c_void_p)]


class gtr_rs_verify(C.Structure):
    _fields_ = [("mat", C.c_void_p), ("am", C.c_void_p), ("macro", C.c_void_p)]


def cfg(mode=SPMD, placement=PL_STACK, fold=1, thread_limit=256, num_teams=0, smem_stack_bytes=0, flags=0):
    return gtr_launch_cfg(num_teams, thread_limit, mode, placement, fold, smem_stack_bytes, flags)


# ---------------------------------------------------------------- prototypes
_i, _u, _i64, _u64, _vp = C.c_int, C.c_uint32, C.c_int64, C.c_uint64, C.c_void_p
_P = C.POINTER
_proto = {
    "gtr_version": (_i, []),
    "gtr_strerror": (C.c_char_p, [_i]),
    "gtr_ctx_create": (_i, [_i, _vp, _u64, _P(_vp)]),
    "gtr_ctx_destroy": (_i, [_vp]),
    "gtr_ctx_check": (_i, [_vp, _vp]),
    "gtr_ctx_fallback_high_water": (_i, [_vp, C.POINTER(C.c_uint64), C.c_int32, _vp]),
    "gtr_ctx_set_spin_limit": (_i, [_vp, _u64]),
    "gtr_watchdog_selftest": (_i, [_vp, C.c_int32, _vp]),
    "gtr_query_variant": (_i, [_i, _P(gtr_launch_cfg), _P(gtr_variant_info)]),
    "gtr_forkjoin": (_i, [_vp, _P(gtr_launch_cfg), _i64, C.c_int32, C.c_int32, _vp, _vp]),
    "gtr_barrier_floor": (_i, [_vp, _P(gtr_launch_cfg), _i64, _vp, _vp]),
    "gtr_fp64_probe": (_i, [_vp, _i64, _vp, _P(C.c_double), _vp]),
    "gtr_ddiv_selftest": (_i, [_vp, _u64, _u64, _vp, _vp]),
    "gtr_semantics": (_i, [_vp, _P(gtr_launch_cfg), C.c_int32, _vp, _i64, _vp]),
    "gtr_xs_build_workspace_bytes": (_u64, [_i64, _i64]),
    "gtr_xs_build_egrid": (_i, [_vp, _vp, _i64, _i64, _vp, _vp, _vp]),
    "gtr_xs_build_index_grid": (_i, [_vp, _vp, _i64, _i64, _vp, _vp, _vp, _vp]),
    "gtr_xs_build_energies": (_i, [_vp, _vp, _i64, _i64, _vp, _vp]),
    "gtr_xs_build_hash_grid": (_i, [_vp, _vp, _i64, _i64, C.c_int32, _vp, _vp]),
    "gtr_xs_build_union_bins": (_i, [_vp, _vp, _i64, C.c_int32, _vp, _vp]),
    "gtr_rs_build_wide_poles": (_i, [_vp, _vp, _i64, _vp, _vp]),
    "gtr_xs_lookup": (_i, [_vp, _P(gtr_launch_cfg), _P(gtr_xs_tables), _u64, _u64, _u64, _vp,
                           _P(gtr_xs_verify), _vp]),
    "gtr_xs_sorted_workspace_bytes": (_u64, [_u64]),
    "gtr_xs_lookup_sorted": (_i, [_vp, _P(gtr_launch_cfg), _P(gtr_xs_tables), _u64, _u64, _u64, _vp,
                                  _P(gtr_xs_verify), _vp, _u64, _vp]),
    "gtr_xs_sort_lookups": (_i, [_vp, _P(gtr_xs_tables), _u64, _u64, _u64, _vp, _u64, _vp]),
    "gtr_xs_lookup_presorted": (_i, [_vp, _P(gtr_launch_cfg), _P(gtr_xs_tables), _u64, _u64, _vp,
                                     _P(gtr_xs_verify), _vp, _u64, _vp]),
    "gtr_xs_lookup_peers": (_i, [_vp, _P(gtr_launch_cfg), _P(gtr_xs_tables), _u64, _u64, _u64, _P(_u64), C.c_int32,
                                 _vp]),
    "gtr_xs_lookup_host": (_i, [_vp, _P(gtr_launch_cfg), _P(gtr_xs_tables), _P(gtr_xs_request), _vp, _vp]),
    "gtr_xs_lookup_presorted_peers": (_i, [_vp, _P(gtr_launch_cfg), _P(gtr_xs_tables), _u64, _u64, _P(_u64),
                                           C.c_int32, _vp, _u64, _vp]),
    "gtr_xs_lookup_sorted_host": (_i, [_vp, _P(gtr_launch_cfg), _P(gtr_xs_tables), _P(gtr_xs_request), _vp, _vp,
                                       _u64, _vp]),
    "gtr_l2_persist": (_i, [_vp, _vp, _u64, _u64, C.c_float, _vp]),
    "gtr_su3_mat_nn": (_i, [_vp, _P(gtr_launch_cfg), _vp, _vp, _vp, _i64, C.c_int32, _vp]),
    "gtr_rs_lookup": (_i, [_vp, _P(gtr_launch_cfg), _P(gtr_rs_tables), _u64, _u64, _u64, _vp,
                           _P(gtr_rs_verify), _vp]),
}
for _n, (_r, _a) in _proto.items():
    _f = getattr(_lib, _n)
    _f.restype, _f.argtypes = _r, _a

EXPORTED = tuple(_proto)


def _ptr(x):
    if x is None:
        return None
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    return int(x)


def _stream(s):
    if s is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if hasattr(s, "cuda_stream"):
        return s.cuda_stream
    return int(s)


def _check(fn, st):
    if st != GTR_OK:
        raise GtrError(fn, st)
    return st


# ---------------------------------------------------------------- API
def gtr_version():
    return _lib.gtr_version()


def gtr_strerror(status):
    return _lib.gtr_strerror(status).decode()


def gtr_ctx_create(device=0, fallback_pool=None, fallback_pool_bytes=0):
    h = _vp()
    _check("gtr_ctx_create", _lib.gtr_ctx_create(device, _ptr(fallback_pool), fallback_pool_bytes, C.byref(h)))
    return h


def gtr_ctx_destroy(ctx):
    return _check("gtr_ctx_destroy", _lib.gtr_ctx_destroy(ctx))


def gtr_ctx_check(ctx, stream=None, raise_on_error=True):
    st = _lib.gtr_ctx_check(ctx, _stream(stream))
    return _check("gtr_ctx_check", st) if raise_on_error else st


def gtr_ctx_fallback_high_water(ctx, reset=False, stream=None):
    """Largest bytes of globalized variables one thread held in the global
    fallback pool since creation / the last reset."""
    v = C.c_uint64(0)
    _check("gtr_ctx_fallback_high_water", _lib.gtr_ctx_fallback_high_water(ctx, C.byref(v), 1 if reset else 0,
                                                                            _stream(stream)))
    return int(v.value)


def gtr_ctx_set_spin_limit(ctx, polls):
    """Watchdog: polls of a runtime spin-wait before it sets the hang bit (0: default)."""
    return _check("gtr_ctx_set_spin_limit", _lib.gtr_ctx_set_spin_limit(ctx, polls))


def gtr_watchdog_selftest(ctx, kind, stream=None):
    """Enqueue a kernel whose waits never complete (0: software barrier, 1: mbarrier)."""
    return _check("gtr_watchdog_selftest", _lib.gtr_watchdog_selftest(ctx, kind, _stream(stream)))


def gtr_query_variant(kernel, launch_cfg):
    info = gtr_variant_info()
    _check("gtr_query_variant", _lib.gtr_query_variant(kernel, C.byref(launch_cfg), C.byref(info)))
    return {k: getattr(info, k) for k, _ in gtr_variant_info._fields_}


def gtr_forkjoin(ctx, launch_cfg, regions, body, n_distinct, d_out, stream=None):
    return _check("gtr_forkjoin", _lib.gtr_forkjoin(ctx, C.byref(launch_cfg), regions, body, n_distinct,
                                                    _ptr(d_out), _stream(stream)))


def gtr_barrier_floor(ctx, launch_cfg, iters, d_out, stream=None):
    return _check("gtr_barrier_floor", _lib.gtr_barrier_floor(ctx, C.byref(launch_cfg), iters, _ptr(d_out),
                                                              _stream(stream)))


def gtr_ddiv_selftest(ctx, n, seed, d_counts, stream=None):
    return _check("gtr_ddiv_selftest", _lib.gtr_ddiv_selftest(ctx, n, seed, _ptr(d_counts), _stream(stream)))


def gtr_fp64_probe(ctx, iters, d_out, stream=None):
    """Launch the fp64 FMA probe; returns the flops of one launch."""
    f = C.c_double()
    _check("gtr_fp64_probe", _lib.gtr_fp64_probe(ctx, iters, _ptr(d_out), C.byref(f), _stream(stream)))
    return f.value


def gtr_semantics(ctx, launch_cfg, test_id, d_out, out_len, stream=None):
    return _check("gtr_semantics", _lib.gtr_semantics(ctx, C.byref(launch_cfg), test_id, _ptr(d_out), out_len,
                                                      _stream(stream)))


def gtr_xs_build_workspace_bytes(n_iso, n_gp):
    return _lib.gtr_xs_build_workspace_bytes(n_iso, n_gp)


def gtr_xs_build_egrid(ctx, d_grid, n_iso, n_gp, d_egrid_out, d_workspace, stream=None):
    return _check("gtr_xs_build_egrid", _lib.gtr_xs_build_egrid(ctx, _ptr(d_grid), n_iso, n_gp, _ptr(d_egrid_out),
                                                                _ptr(d_workspace), _stream(stream)))


def gtr_xs_build_energies(ctx, d_grid, n_iso, n_gp, d_energies_out, stream=None):
    return _check("gtr_xs_build_energies", _lib.gtr_xs_build_energies(ctx, _ptr(d_grid), n_iso, n_gp,
                                                                      _ptr(d_energies_out), _stream(stream)))


def gtr_xs_build_hash_grid(ctx, d_energies, n_iso, n_gp, hash_bins, d_hash_out, stream=None):
    return _check("gtr_xs_build_hash_grid", _lib.gtr_xs_build_hash_grid(ctx, _ptr(d_energies), n_iso, n_gp,
                                                                        hash_bins, _ptr(d_hash_out),
                                                                        _stream(stream)))


def gtr_xs_build_union_bins(ctx, d_egrid, n_union, log2_bins, d_bins_out, stream=None):
    return _check("gtr_xs_build_union_bins", _lib.gtr_xs_build_union_bins(ctx, _ptr(d_egrid), n_union, log2_bins,
                                                                          _ptr(d_bins_out), _stream(stream)))


def gtr_rs_build_wide_poles(ctx, d_poles, n_records, d_out, stream=None):
    return _check("gtr_rs_build_wide_poles", _lib.gtr_rs_build_wide_poles(ctx, _ptr(d_poles), n_records, _ptr(d_out),
                                                                          _stream(stream)))


def gtr_xs_build_index_grid(ctx, d_grid, n_iso, n_gp, d_egrid, d_index_out, d_workspace, stream=None):
    return _check("gtr_xs_build_index_grid",
                  _lib.gtr_xs_build_index_grid(ctx, _ptr(d_grid), n_iso, n_gp, _ptr(d_egrid), _ptr(d_index_out),
                                               _ptr(d_workspace), _stream(stream)))


def gtr_xs_lookup(ctx, launch_cfg, tables, first, n, seed, d_out, verify=None, stream=None):
    return _check("gtr_xs_lookup", _lib.gtr_xs_lookup(ctx, C.byref(launch_cfg), C.byref(tables), first, n, seed,
                                                      _ptr(d_out), C.byref(verify) if verify else None,
                                                      _stream(stream)))


def gtr_xs_sorted_workspace_bytes(n):
    return _lib.gtr_xs_sorted_workspace_bytes(n)


def gtr_xs_lookup_sorted(ctx, launch_cfg, tables, first, n, seed, d_out, d_workspace, verify=None, stream=None):
    """d_workspace: a device tensor of at least gtr_xs_sorted_workspace_bytes(n) bytes."""
    nbytes = d_workspace.numel() * d_workspace.element_size()
    return _check("gtr_xs_lookup_sorted",
                  _lib.gtr_xs_lookup_sorted(ctx, C.byref(launch_cfg), C.byref(tables), first, n, seed, _ptr(d_out),
                                            C.byref(verify) if verify else None, _ptr(d_workspace), nbytes,
                                            _stream(stream)))


def gtr_xs_lookup_peers(ctx, launch_cfg, tables, first, n, seed, peer_ptrs, stream=None):
    """peer_ptrs: device addresses (ints) of every rank's 18-u64 result buffer."""
    arr = (_u64 * len(peer_ptrs))(*peer_ptrs)
    return _check("gtr_xs_lookup_peers",
                  _lib.gtr_xs_lookup_peers(ctx, C.byref(launch_cfg), C.byref(tables), first, n, seed, arr,
                                           len(peer_ptrs), _stream(stream)))


def gtr_xs_lookup_host(ctx, launch_cfg, tables, h_req, h_out, stream=None):
    return _check("gtr_xs_lookup_host", _lib.gtr_xs_lookup_host(ctx, C.byref(launch_cfg), C.byref(tables),
                                                                C.byref(h_req), _ptr(h_out), _stream(stream)))


def gtr_xs_sort_lookups(ctx, tables, first, n, seed, d_workspace, stream=None):
    nbytes = d_workspace.numel() * d_workspace.element_size()
    return _check("gtr_xs_sort_lookups",
                  _lib.gtr_xs_sort_lookups(ctx, C.byref(tables), first, n, seed, _ptr(d_workspace), nbytes,
                                           _stream(stream)))


def gtr_xs_lookup_presorted(ctx, launch_cfg, tables, first, n, d_out, d_workspace, verify=None, stream=None):
    nbytes = d_workspace.numel() * d_workspace.element_size()
    return _check("gtr_xs_lookup_presorted",
                  _lib.gtr_xs_lookup_presorted(ctx, C.byref(launch_cfg), C.byref(tables), first, n, _ptr(d_out),
                                               C.byref(verify) if verify else None, _ptr(d_workspace), nbytes,
                                               _stream(stream)))


def gtr_xs_lookup_presorted_peers(ctx, launch_cfg, tables, first, n, peer_ptrs, d_workspace, stream=None):
    arr = (_u64 * len(peer_ptrs))(*peer_ptrs)
    nbytes = d_workspace.numel() * d_workspace.element_size()
    return _check("gtr_xs_lookup_presorted_peers",
                  _lib.gtr_xs_lookup_presorted_peers(ctx, C.byref(launch_cfg), C.byref(tables), first, n, arr,
                                                     len(peer_ptrs), _ptr(d_workspace), nbytes, _stream(stream)))


def gtr_xs_lookup_sorted_host(ctx, launch_cfg, tables, h_req, h_out, d_workspace, stream=None):
    nbytes = d_workspace.numel() * d_workspace.element_size()
    return _check("gtr_xs_lookup_sorted_host",
                  _lib.gtr_xs_lookup_sorted_host(ctx, C.byref(launch_cfg), C.byref(tables), C.byref(h_req),
                                                 _ptr(h_out), _ptr(d_workspace), nbytes, _stream(stream)))


def gtr_su3_mat_nn(ctx, launch_cfg, d_A, d_B, d_C, sites, iters, stream=None):
    return _check("gtr_su3_mat_nn", _lib.gtr_su3_mat_nn(ctx, C.byref(launch_cfg), _ptr(d_A), _ptr(d_B), _ptr(d_C),
                                                        sites, iters, _stream(stream)))


def gtr_rs_lookup(ctx, launch_cfg, tables, first, n, seed, d_out, verify=None, stream=None):
    return _check("gtr_rs_lookup", _lib.gtr_rs_lookup(ctx, C.byref(launch_cfg), C.byref(tables), first, n, seed,
                                                      _ptr(d_out), C.byref(verify) if verify else None,
                                                      _stream(stream)))


def gtr_l2_persist(ctx, d_base, nbytes, persist_bytes, hit_ratio, stream=None):
    return _check("gtr_l2_persist", _lib.gtr_l2_persist(ctx, _ptr(d_base), nbytes, persist_bytes, hit_ratio,
                                                        _stream(stream)))

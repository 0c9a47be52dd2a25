"""Device-resident problems: upload the generator's tables with PyTorch (device
memory only) and build the XS acceleration structures with libgtr's own
kernels.  Plumbing -- no arithmetic of the method happens in Python.
"""
import numpy as np
import torch

from . import gtr as G


def _dev(a, device):
    return torch.from_numpy(np.ascontiguousarray(a)).to(device, non_blocking=False)


class XsDevice:
    """XS tables on the GPU: the nuclide grid (uploaded) and the acceleration
    structure of `grid_type`, built by libgtr: unionized energy grid + index
    grid (gtr_xs_build_egrid / _index_grid), or the compact per-nuclide
    energies (+ the hash grid) for the nuclide / hash grid types.

    `union_bins_log2` (identical results, on by
    default): a bin table narrowing the union search (None: the plain
    full-range binary search)."""

    def __init__(self, ctx, t, device="cuda", stream=None, grid_type=0, hash_bins=10000, union_bins_log2=21):
        self.n_iso, self.n_gp = int(t["n_iso"]), int(t["n_gp"])
        self.n_union = self.n_iso * self.n_gp
        self.grid_type, self.hash_bins = grid_type, hash_bins
        self.grid = _dev(t["grid"], device)
        self.num_nucs = _dev(t["num_nucs"].astype(np.int32), device)
        self.mats = _dev(t["mats"].astype(np.int32), device)
        self.concs = _dev(t["concs"].astype(np.float64), device)
        self.max_num_nucs = int(t["mats"].shape[1])
        self.egrid = self.index_grid = self.energies = self.hash_index = None
        if grid_type == G.XS_UNIONIZED:
            self.egrid = torch.empty(self.n_union, dtype=torch.float64, device=device)
            self.index_grid = torch.empty((self.n_union, self.n_iso), dtype=torch.int32, device=device)
            ws = torch.empty(G.gtr_xs_build_workspace_bytes(self.n_iso, self.n_gp), dtype=torch.uint8,
                             device=device)
            G.gtr_xs_build_egrid(ctx, self.grid, self.n_iso, self.n_gp, self.egrid, ws, stream)
            G.gtr_xs_build_index_grid(ctx, self.grid, self.n_iso, self.n_gp, self.egrid, self.index_grid, ws,
                                      stream)
            del ws
        else:
            self.energies = torch.empty((self.n_iso, self.n_gp), dtype=torch.float64, device=device)
            G.gtr_xs_build_energies(ctx, self.grid, self.n_iso, self.n_gp, self.energies, stream)
            if grid_type == G.XS_HASH:
                self.hash_index = torch.empty((hash_bins, self.n_iso), dtype=torch.int32, device=device)
                G.gtr_xs_build_hash_grid(ctx, self.energies, self.n_iso, self.n_gp, hash_bins, self.hash_index,
                                         stream)
        self.union_bins, self.union_bins_log2 = None, 0
        if grid_type == G.XS_UNIONIZED and union_bins_log2 is not None:
            self.union_bins_log2 = int(union_bins_log2)
            self.union_bins = torch.empty((1 << self.union_bins_log2) + 1, dtype=torch.int32, device=device)
            G.gtr_xs_build_union_bins(ctx, self.egrid, self.n_union, self.union_bins_log2, self.union_bins, stream)
        G.gtr_ctx_check(ctx, stream)           # unsorted or NaN energies -> GtrError
        p = lambda x: x.data_ptr() if x is not None else None   # noqa: E731
        self.tables = G.gtr_xs_tables(self.n_iso, self.n_gp, self.n_union, self.max_num_nucs,
                                      p(self.egrid), p(self.index_grid), self.grid.data_ptr(),
                                      self.num_nucs.data_ptr(), self.mats.data_ptr(), self.concs.data_ptr(),
                                      grid_type, hash_bins, p(self.hash_index), p(self.energies),
                                      p(self.union_bins), self.union_bins_log2)

    def nbytes(self):
        return sum(x.numel() * x.element_size() for x in
                   (self.grid, self.egrid, self.index_grid, self.energies, self.hash_index, self.num_nucs,
                    self.mats, self.concs, self.union_bins) if x is not None)

    def verify_buffers(self, n, device="cuda"):
        bufs = {"mat": torch.zeros(n, dtype=torch.uint8, device=device),
                "u": torch.zeros(n, dtype=torch.int32, device=device),
                "am": torch.zeros(n, dtype=torch.uint8, device=device),
                "macro": torch.zeros((n, 5), dtype=torch.float64, device=device)}
        v = G.gtr_xs_verify(bufs["mat"].data_ptr(), bufs["u"].data_ptr(), bufs["am"].data_ptr(),
                            bufs["macro"].data_ptr())
        return v, bufs


class RsDevice:
    """RS tables on the GPU.  `wide_poles` (on by default; identical results):
    also build the 96-byte pole records (gtr_rs_build_wide_poles) the lookups
    then read with 256-bit loads; False keeps RSBench's 72-byte records."""

    def __init__(self, t, device="cuda", ctx=None, wide_poles=True, stream=None):
        self.n_windows = _dev(t["n_windows"].astype(np.int32), device)
        self.poles = _dev(np.ascontiguousarray(t["poles"]).view(np.uint8), device)
        self.windows = _dev(np.ascontiguousarray(t["windows"]).view(np.uint8), device)
        self.k0rs = _dev(t["k0rs"].astype(np.float64), device)
        self.num_nucs = _dev(t["num_nucs"].astype(np.int32), device)
        self.mats = _dev(t["mats"].astype(np.int32), device)
        self.concs = _dev(t["concs"].astype(np.float64), device)
        self.poles_wide = None
        if wide_poles:
            own = ctx is None
            c = G.gtr_ctx_create(torch.device(device).index or 0) if own else ctx
            n_rec = int(t["n_nuc"]) * int(t["max_poles"])
            self.poles_wide = torch.empty((n_rec, 12), dtype=torch.float64, device=device)
            G.gtr_rs_build_wide_poles(c, self.poles, n_rec, self.poles_wide, stream)
            G.gtr_ctx_check(c, stream)
            if own:
                G.gtr_ctx_destroy(c)
        self.tables = G.gtr_rs_tables(int(t["n_nuc"]), int(t["max_poles"]), int(t["max_windows"]),
                                      int(t["mats"].shape[1]), self.n_windows.data_ptr(), self.poles.data_ptr(),
                                      self.windows.data_ptr(), self.k0rs.data_ptr(), self.num_nucs.data_ptr(),
                                      self.mats.data_ptr(), self.concs.data_ptr(),
                                      self.poles_wide.data_ptr() if self.poles_wide is not None else None)

    def verify_buffers(self, n, device="cuda"):
        bufs = {"mat": torch.zeros(n, dtype=torch.uint8, device=device),
                "am": torch.zeros(n, dtype=torch.uint8, device=device),
                "macro": torch.zeros((n, 4), dtype=torch.float64, device=device)}
        v = G.gtr_rs_verify(bufs["mat"].data_ptr(), bufs["am"].data_ptr(), bufs["macro"].data_ptr())
        return v, bufs


def su3_device(A, B, device="cuda"):
    """complex128 numpy arrays -> float64 device tensors [..., 2] (same bytes)."""
    dA = _dev(np.ascontiguousarray(A).view(np.float64), device)
    dB = _dev(np.ascontiguousarray(B).view(np.float64), device)
    return dA, dB

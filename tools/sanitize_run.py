"""Small launches of every runtime mode x placement for compute-sanitizer
(memcheck / racecheck / synccheck / initcheck):

    compute-sanitizer --tool racecheck python tools/sanitize_run.py [part ...]

parts (default: all): fj sem xs xs_grids xs_sorted xs_peers su3 su3_tma rs
Covers GENERIC / CASCADE / CSM / SPMD (+ NATIVE where the family has it) x the
five placements (RUNTIME, GLOBAL, SHARED_STATIC, STACK, COALESCED), folded and
not, the semantic programs 0-8 (6-8: ICVs, soft barriers of partial teams),
XS bucketed / plain / history / sorted / nuclide + hash grids / the fused
peer-combine epilogue, SU3 plain and tile-streamed (GTR_F_TMA: mbarriers +
bulk copies), RS wide and narrow pole records.
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch  # noqa: E402

import gtr_inputs.rs as RS  # noqa: E402
import gtr_inputs.su3 as S  # noqa: E402
import gtr_inputs.xs as X  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice, XsDevice, su3_device  # noqa: E402

parts = set(sys.argv[1:]) or {"fj", "sem", "xs", "xs_grids", "xs_sorted", "xs_peers", "su3", "su3_tma", "rs"}
pool = torch.zeros(16 << 20, dtype=torch.uint8, device="cuda")
ctx = G.gtr_ctx_create(0, pool.data_ptr(), pool.numel())
modes = (G.GENERIC, G.GENERIC_CASCADE, G.CSM, G.SPMD)
pls = (G.PL_RUNTIME, G.PL_GLOBAL, G.PL_SHARED_STATIC, G.PL_STACK, G.PL_COALESCED)
teams = 2
ran = []


def u64(n):
    return torch.zeros(n, dtype=torch.uint64, device="cuda")


if "fj" in parts:
    for m in modes:
        for p in pls:
            for fold in (0, 1):
                for body, K in ((0, 1), (1, 3), (2, 3)):
                    G.gtr_forkjoin(ctx, G.cfg(m, p, fold, 128, num_teams=teams), 6, body, K, u64(teams))
    for p in pls:          # one-warp teams (warp-team guards) and the 1-barrier broadcast
        G.gtr_forkjoin(ctx, G.cfg(G.SPMD, p, 1, 32, num_teams=teams), 6, 2, 3, u64(teams))
        G.gtr_forkjoin(ctx, G.cfg(G.SPMD, p, 1, 128, num_teams=teams, flags=G.F_BCAST_1BAR), 6, 2, 3, u64(teams))
    ran.append("fj")
if "sem" in parts:
    for m in modes:
        for p in pls:
            for t in range(9):
                G.gtr_semantics(ctx, G.cfg(m, p, 0, 64, num_teams=teams), t, u64(8192), 8192)
            for t in range(5):
                G.gtr_semantics(ctx, G.cfg(m, p, 1, 64, num_teams=teams), t, u64(8192), 8192)
    ran.append("sem")
G.gtr_ctx_check(ctx)
if parts & {"xs", "xs_grids", "xs_sorted", "xs_peers"}:
    tx = X.make_tables(8, 40)
    xs = XsDevice(ctx, tx)
    if "xs" in parts:
        for m in modes:
            for p in pls:
                for flags in (0, G.F_PLAIN, G.F_HISTORY):
                    G.gtr_xs_lookup(ctx, G.cfg(m, p, 0, 128, num_teams=teams, flags=flags), xs.tables, 0, 3000,
                                    X.SEED_L, u64(18))
        for m in (G.CSM, G.SPMD):      # the headline kernels (CSM register-capped), union bins on
            for nt in (128, 256):
                G.gtr_xs_lookup(ctx, G.cfg(m, G.PL_STACK, 1, nt, num_teams=teams), xs.tables, 0, 3000, X.SEED_L,
                                u64(18))
        for flags in (0, G.F_HISTORY):
            G.gtr_xs_lookup(ctx, G.cfg(G.NATIVE, G.PL_STACK, 1, 128, num_teams=teams, flags=flags), xs.tables, 0,
                            3000, X.SEED_L, u64(18))
        ran.append("xs")
    if "xs_grids" in parts:
        for gt in (G.XS_NUCLIDE, G.XS_HASH):
            xg = XsDevice(ctx, tx, grid_type=gt, hash_bins=97)
            for m, p, f in ((G.SPMD, G.PL_STACK, 1), (G.GENERIC, G.PL_RUNTIME, 0), (G.NATIVE, G.PL_STACK, 1)):
                G.gtr_xs_lookup(ctx, G.cfg(m, p, f, 128, num_teams=teams), xg.tables, 0, 2000, X.SEED_L, u64(18))
        ran.append("xs_grids")
    if "xs_sorted" in parts:
        ws = torch.empty(G.gtr_xs_sorted_workspace_bytes(3000), dtype=torch.uint8, device="cuda")
        for m, p, f, fl, nt in ((G.SPMD, G.PL_STACK, 1, 0, 128), (G.CSM, G.PL_RUNTIME, 0, 0, 128),
                                (G.GENERIC, G.PL_STACK, 1, 0, 128), (G.SPMD, G.PL_STACK, 1, G.F_PLAIN, 128),
                                (G.NATIVE, G.PL_STACK, 1, 0, 128), (G.SPMD, G.PL_STACK, 1, 0, 256),
                                (G.CSM, G.PL_STACK, 1, 0, 256), (G.NATIVE, G.PL_STACK, 1, G.F_NATIVE_BUCKETED, 256)):
            G.gtr_xs_lookup_sorted(ctx, G.cfg(m, p, f, nt, num_teams=teams, flags=fl), xs.tables, 0, 3000, X.SEED_L,
                                   u64(18), ws)
        # the split form and the host-request form (warp-coherent path on a
        # denser table: 68 nuclides x 200 gridpoints, 20,000 lookups)
        td = X.make_tables(68, 200)
        xd = XsDevice(ctx, td)
        wd = torch.empty(G.gtr_xs_sorted_workspace_bytes(20000), dtype=torch.uint8, device="cuda")
        G.gtr_xs_sort_lookups(ctx, xd.tables, 5, 20000, X.SEED_L, wd)
        G.gtr_xs_lookup_presorted(ctx, G.cfg(G.SPMD, G.PL_STACK, 1, 256, num_teams=teams), xd.tables, 5, 20000,
                                  u64(18), wd)
        G.gtr_xs_lookup_presorted_peers(ctx, G.cfg(G.CSM, G.PL_STACK, 1, 128, num_teams=teams), xd.tables, 5, 20000,
                                        [u64(18).data_ptr()], wd)
        h = torch.zeros(18, dtype=torch.uint64).pin_memory()
        G.gtr_xs_lookup_sorted_host(ctx, G.cfg(G.SPMD, G.PL_STACK, 1, 256, num_teams=teams), xd.tables,
                                    G.gtr_xs_request(0, 20000, X.SEED_L), h, wd)
        # duplicate gridpoint energies: union scatter + sequential-rule index builder
        tdup = X.make_tables(3, 50)
        tdup["grid"][0, 11, 0] = tdup["grid"][0, 10, 0]
        tdup["grid"][1, 30, 0] = tdup["grid"][0, 30, 0]
        for n_ in range(3):
            tdup["grid"][n_] = tdup["grid"][n_][np.argsort(tdup["grid"][n_, :, 0], kind="stable")]
        XsDevice(ctx, tdup)
        ran.append("xs_sorted")
    if "xs_peers" in parts:
        bufs = [u64(18) for _ in range(3)]
        for m in (G.SPMD, G.CSM, G.NATIVE):
            G.gtr_xs_lookup_peers(ctx, G.cfg(m, G.PL_STACK, 1, 128, num_teams=teams), xs.tables, 0, 3000, X.SEED_L,
                                  [b.data_ptr() for b in bufs])
        ran.append("xs_peers")
G.gtr_ctx_check(ctx)
if parts & {"su3", "su3_tma"}:
    A, B = S.make_lattice(40, "random")
    dA, dB = su3_device(A, B)
    dC = torch.empty_like(dA)
    if "su3" in parts:
        for m in modes:
            for p in pls:
                G.gtr_su3_mat_nn(ctx, G.cfg(m, p, 0, 64, num_teams=teams), dA, dB, dC, 40, 1)
        G.gtr_su3_mat_nn(ctx, G.cfg(G.NATIVE, G.PL_STACK, 1, 128, num_teams=teams), dA, dB, dC, 40, 1)
        ran.append("su3")
    if "su3_tma" in parts:
        for m in modes:
            for p in (G.PL_RUNTIME, G.PL_STACK, G.PL_COALESCED):
                G.gtr_su3_mat_nn(ctx, G.cfg(m, p, 0, 64, num_teams=teams, flags=G.F_TMA), dA, dB, dC, 40, 1)
        G.gtr_su3_mat_nn(ctx, G.cfg(G.NATIVE, G.PL_STACK, 1, 128, num_teams=teams, flags=G.F_TMA), dA, dB, dC, 40, 1)
        ran.append("su3_tma")
G.gtr_ctx_check(ctx)
if "rs" in parts:
    trs = RS.make_tables(n_nuc=20, avg_poles=40, avg_windows=5)
    for wide in (True, False):
        rs = RsDevice(trs, ctx=ctx, wide_poles=wide)
        for m in modes:
            for p in pls:
                G.gtr_rs_lookup(ctx, G.cfg(m, p, 0, 128, num_teams=teams), rs.tables, 0, 700, X.SEED_L, u64(18))
        for m in modes:
            G.gtr_rs_lookup(ctx, G.cfg(m, G.PL_STACK, 1, 128, num_teams=teams, flags=G.F_PLAIN), rs.tables, 0, 700,
                            X.SEED_L, u64(18))
        G.gtr_rs_lookup(ctx, G.cfg(G.NATIVE, G.PL_STACK, 1, 128, num_teams=teams), rs.tables, 0, 700, X.SEED_L, u64(18))
    ran.append("rs")
G.gtr_ctx_check(ctx)
print("sanitize run ok:", " ".join(ran))

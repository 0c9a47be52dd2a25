"""Small launches of every runtime mode for compute-sanitizer
(memcheck / racecheck / synccheck):

    compute-sanitizer --tool racecheck python tools/sanitize_run.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gtr_inputs.rs as RS  # noqa: E402
import gtr_inputs.su3 as S  # noqa: E402
import gtr_inputs.xs as X  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice, XsDevice, su3_device  # noqa: E402

pool = torch.zeros(16 << 20, dtype=torch.uint8, device="cuda")
ctx = G.gtr_ctx_create(0, pool.data_ptr(), pool.numel())
modes = (G.GENERIC, G.GENERIC_CASCADE, G.CSM, G.SPMD)
pls = (G.PL_RUNTIME, G.PL_SHARED_STATIC, G.PL_STACK)
teams = 2
for m in modes:
    for p in pls:
        for body in (0, 1, 2):
            out = torch.zeros(teams, dtype=torch.uint64, device="cuda")
            G.gtr_forkjoin(ctx, G.cfg(m, p, 0, 128, num_teams=teams), 6, body, 3, out)
        for t in range(6):
            out = torch.zeros(4096, dtype=torch.uint64, device="cuda")
            G.gtr_semantics(ctx, G.cfg(m, p, 0, 64, num_teams=teams), t, out, out.numel())
G.gtr_ctx_check(ctx)
xs = XsDevice(ctx, X.make_tables(8, 40))
for m in modes + (G.NATIVE,):
    for flags in (0, G.F_PLAIN):
        out = torch.zeros(18, dtype=torch.uint64, device="cuda")
        G.gtr_xs_lookup(ctx, G.cfg(m, G.PL_STACK if m == G.NATIVE else G.PL_RUNTIME, 0, 128, num_teams=teams,
                                   flags=flags), xs.tables, 0, 3000, X.SEED_L, out)
for m in (G.CSM, G.SPMD):      # the headline kernels (CSM register-capped), union bins on
    for nt in (128, 256):
        out = torch.zeros(18, dtype=torch.uint64, device="cuda")
        G.gtr_xs_lookup(ctx, G.cfg(m, G.PL_STACK, 1, nt, num_teams=teams), xs.tables, 0, 3000, X.SEED_L, out)
A, B = S.make_lattice(40, "random")
dA, dB = su3_device(A, B)
dC = torch.empty_like(dA)
for m in modes:
    G.gtr_su3_mat_nn(ctx, G.cfg(m, G.PL_RUNTIME, 0, 64, num_teams=teams), dA, dB, dC, 40, 1)
rs = RsDevice(RS.make_tables(n_nuc=20, avg_poles=40, avg_windows=5))
for m in modes:
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    G.gtr_rs_lookup(ctx, G.cfg(m, G.PL_RUNTIME, 0, 128, num_teams=teams), rs.tables, 0, 700, X.SEED_L, out)
    G.gtr_rs_lookup(ctx, G.cfg(m, G.PL_STACK, 1, 128, num_teams=teams), rs.tables, 0, 700, X.SEED_L, out)
G.gtr_ctx_check(ctx)
print("sanitize run ok")

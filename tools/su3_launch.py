"""Time SU3 mat_nn (32^4, fp64) per variant: ms/iteration and GB/s
(1152 B per site).   python tools/su3_launch.py [--reps 20]"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gtr_inputs.su3 as S  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200.problems import su3_device  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--reps", type=int, default=20)
a = ap.parse_args()
ctx = G.gtr_ctx_create(0)
sites = 32 ** 4
A, B = S.make_lattice(sites, "constant")
dA, dB = su3_device(A, B)
dC = torch.empty_like(dA)
V = [("native256", G.cfg(G.NATIVE, G.PL_STACK, 1, 256)),
     ("native_tma128", G.cfg(G.NATIVE, G.PL_STACK, 1, 128, flags=G.F_TMA)),
     ("native_tma256", G.cfg(G.NATIVE, G.PL_STACK, 1, 256, flags=G.F_TMA)),
     ("native_tma512", G.cfg(G.NATIVE, G.PL_STACK, 1, 512, flags=G.F_TMA)),
     ("spmd64", G.cfg(G.SPMD, G.PL_STACK, 1, 64)),
     ("spmd_tma64", G.cfg(G.SPMD, G.PL_STACK, 1, 64, flags=G.F_TMA)),
     ("spmd_tma128", G.cfg(G.SPMD, G.PL_STACK, 1, 128, flags=G.F_TMA)),
     ("csm_tma64", G.cfg(G.CSM, G.PL_STACK, 1, 64, flags=G.F_TMA)),
     ("csm_tma128", G.cfg(G.CSM, G.PL_STACK, 1, 128, flags=G.F_TMA)),
     ("generic_tma128", G.cfg(G.GENERIC, G.PL_STACK, 1, 128, flags=G.F_TMA))]
for name, c in V:
    G.gtr_su3_mat_nn(ctx, c, dA, dB, dC, sites, 2)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    G.gtr_su3_mat_nn(ctx, c, dA, dB, dC, sites, a.reps)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / a.reps
    ok = bool(torch.all(dC.view(-1, 2)[:, 0] == 1.0).item())
    info = G.gtr_query_variant(G.K_SU3, c)
    print(f"{name:16s} {ms:7.4f} ms  {sites * 1152 / ms / 1e6:7.1f} GB/s  regs {info['regs']} "
          f"teams/SM {info['teams_per_sm']}  ok {ok}", flush=True)
G.gtr_ctx_check(ctx)

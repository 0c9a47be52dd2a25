"""ns per fork/join of the broadcast body (a guarded side effect producing a
value) and of the empty body, SPMD, per thread_limit and
placement; 148 teams (one per SM), 20,000 regions.

    python tools/fj_bcast.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G  # noqa: E402

ctx = G.gtr_ctx_create(0)
R, teams = 20000, 148
fo = torch.zeros(teams, dtype=torch.uint64, device="cuda")


def t(fn, reps=3):
    fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps * 1e6 / R


for nt in (32, 128, 256):
    fl = G.cfg(thread_limit=nt, num_teams=teams)
    row = [f"t{nt} floor {t(lambda: G.gtr_barrier_floor(ctx, fl, R, fo)):6.1f}"]
    for name, m, pl, flags in (("spmd_shared", G.SPMD, G.PL_SHARED_STATIC, 0), ("spmd_stack", G.SPMD, G.PL_STACK, 0),
                               ("spmd_stack_1bar", G.SPMD, G.PL_STACK, G.F_BCAST_1BAR),
                               ("csm_shared", G.CSM, G.PL_SHARED_STATIC, 0), ("generic_shared", G.GENERIC, G.PL_SHARED_STATIC, 0)):
        c = G.cfg(m, pl, 1, nt, num_teams=teams, flags=flags)
        row.append(f"{name}: empty {t(lambda: G.gtr_forkjoin(ctx, c, R, 0, 1, fo)):6.1f} "
                   f"bcast {t(lambda: G.gtr_forkjoin(ctx, c, R, 2, 1, fo)):6.1f}")
    print(" | ".join(row), flush=True)

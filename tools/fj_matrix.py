"""ns per fork/join for modes x placements x body x K (148 teams, one per SM)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G
ctx = G.gtr_ctx_create(0)
R, teams, nt = 20000, 148, int(sys.argv[1]) if len(sys.argv) > 1 else 128
fo = torch.zeros(teams, dtype=torch.uint64, device="cuda")
def t(fn, reps=3):
    fn(); torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / reps * 1e6 / R
fl = G.cfg(thread_limit=nt, num_teams=teams)
print("floor", round(t(lambda: G.gtr_barrier_floor(ctx, fl, R, fo)), 1))
for m in (G.GENERIC, G.GENERIC_CASCADE, G.CSM, G.SPMD):
    row = []
    for pl in (G.PL_SHARED_STATIC, G.PL_STACK):
        for body, K in ((0, 1), (1, 1), (1, 4), (1, 16)):
            c = G.cfg(m, pl, 1, nt, num_teams=teams)
            row.append(f"{G.PL_NAMES[pl][:6]} b{body} K{K}: {t(lambda: G.gtr_forkjoin(ctx, c, R, body, K, fo)):6.1f}")
    print(G.MODE_NAMES[m], " | ".join(row))

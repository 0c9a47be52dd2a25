"""One empty-region fork/join launch per runtime mode (148 teams x 128
threads, R = 20000) -- the kernels the fork/join ncu capture profiles."""
import os
import sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G  # noqa: E402

ctx = G.gtr_ctx_create(0)
fo = torch.zeros(148, dtype=torch.uint64, device="cuda")
body = int(sys.argv[1]) if len(sys.argv) > 1 else 0
for m in (G.GENERIC, G.GENERIC_CASCADE, G.CSM, G.SPMD):
    G.gtr_forkjoin(ctx, G.cfg(m, G.PL_STACK, 1, 128, num_teams=148), 20000, body, 1, fo)
torch.cuda.synchronize()
G.gtr_ctx_check(ctx)
print("ok")

import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G
ctx = G.gtr_ctx_create(0)
m = {"spmd": G.SPMD, "csm": G.CSM, "generic": G.GENERIC}[sys.argv[1]]
fo = torch.zeros(148, dtype=torch.uint64, device="cuda")
G.gtr_forkjoin(ctx, G.cfg(m, G.PL_STACK, 1, 128, num_teams=148), 20000, int(sys.argv[2]), 1, fo)
torch.cuda.synchronize(); print("ok")

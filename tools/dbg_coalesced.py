import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import gtr_inputs.rs as RS, gtr_inputs.xs as X
import oracle
from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G
from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice
pool = torch.zeros(256 << 20, dtype=torch.uint8, device="cuda")
ctx = G.gtr_ctx_create(0, pool.data_ptr(), pool.numel())
t = RS.make_tables(n_nuc=40, avg_poles=100, avg_windows=10)
P = oracle.RsProblem(t); n = int(sys.argv[1]) if len(sys.argv) > 1 else 2000
o, ov, _ = P.run(0, n, X.SEED_L, 4, verify=True)
dev = RsDevice(t)
for teams in (1, 0):
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    v, b = dev.verify_buffers(n)
    G.gtr_rs_lookup(ctx, G.cfg(G.GENERIC, G.PL_COALESCED, 0, 128, num_teams=teams, flags=G.F_PLAIN), dev.tables, 0, n, X.SEED_L, out, v)
    print("check", G.gtr_ctx_check(ctx, raise_on_error=False))
    got = b["macro"].cpu().numpy()
    bad = np.where(np.abs(got - ov["macro"]).max(axis=1) > 1e-9 * np.abs(ov["macro"]).max(axis=1))[0]
    print("teams", teams, "bad lookups", len(bad), bad[:20], "lanes", (bad % 32)[:20], "mats", ov["mat"][bad][:20])
    if len(bad): print(got[bad[0]], ov["macro"][bad[0]])

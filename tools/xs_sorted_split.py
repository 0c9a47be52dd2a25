"""Time the sorted lookup kernel over the fuel prefix of the sorted order vs
all 17M (the sort puts material 0 first): where the kernel's time goes.

    python tools/xs_sorted_split.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gtr_inputs.xs as X  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice  # noqa: E402

ctx = G.gtr_ctx_create(0)
xs = XsDevice(ctx, X.make_tables(355))
n = 17_000_000
ws = torch.empty(G.gtr_xs_sorted_workspace_bytes(n), dtype=torch.uint8, device="cuda")
out = torch.zeros(18, dtype=torch.uint64, device="cuda")
G.gtr_xs_sort_lookups(ctx, xs.tables, 0, n, X.SEED_L, ws)
G.gtr_xs_lookup_presorted(ctx, G.cfg(), xs.tables, 0, n, out, ws)
torch.cuda.synchronize()
fuel = int(out.cpu()[1])                       # material-0 tally = the fuel prefix length
c = G.cfg(G.SPMD, G.PL_STACK, 1, 256)
for name, m in (("all", n), ("fuel prefix", fuel), ("first 4M", 4_000_000), ("first 8M", 8_000_000)):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    G.gtr_xs_lookup_presorted(ctx, c, xs.tables, 0, m, out, ws)
    e0.record()
    for _ in range(5):
        G.gtr_xs_lookup_presorted(ctx, c, xs.tables, 0, m, out, ws)
    e1.record()
    torch.cuda.synchronize()
    print(f"{name:12s} {m:9d} lookups  {e0.elapsed_time(e1) / 5:7.3f} ms", flush=True)
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5):
    G.gtr_xs_sort_lookups(ctx, xs.tables, 0, n, X.SEED_L, ws)
e1.record()
torch.cuda.synchronize()
print(f"sort         {n:9d} lookups  {e0.elapsed_time(e1) / 5:7.3f} ms")

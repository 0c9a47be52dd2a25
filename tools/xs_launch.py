"""Launch / time the XS-large lookup per variant (ncu captures and A/B timing).

    python tools/xs_launch.py spmd native ... [--n 17000000] [--reps 3] [--time]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gtr_inputs.xs as X  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice  # noqa: E402

VARIANTS = {
    "native": G.cfg(G.NATIVE, G.PL_STACK, 1, 256),
    "native_bucketed": G.cfg(G.NATIVE, G.PL_STACK, 1, 256, flags=G.F_NATIVE_BUCKETED),
    "native_2teams": G.cfg(G.NATIVE, G.PL_STACK, 1, 256, num_teams=296),   # the SPMD kernel's occupancy
    "spmd_plain_t128": G.cfg(G.SPMD, G.PL_STACK, 1, 128, flags=G.F_PLAIN),
    "native_t128": G.cfg(G.NATIVE, G.PL_STACK, 1, 128),
    "csm_plain": G.cfg(G.CSM, G.PL_STACK, 1, 256, flags=G.F_PLAIN),
    "spmd": G.cfg(G.SPMD, G.PL_STACK, 1, 256),
    "spmd128": G.cfg(G.SPMD, G.PL_STACK, 1, 128),
    "spmd_shared": G.cfg(G.SPMD, G.PL_SHARED_STATIC, 1, 256),
    "spmd_plain": G.cfg(G.SPMD, G.PL_STACK, 1, 256, flags=G.F_PLAIN),
    "spmd_runtime": G.cfg(G.SPMD, G.PL_RUNTIME, 0, 256),
    "csm": G.cfg(G.CSM, G.PL_STACK, 1, 256),
    "csm128": G.cfg(G.CSM, G.PL_STACK, 1, 128),
    "generic": G.cfg(G.GENERIC, G.PL_STACK, 1, 256),
    "spmd_history": G.cfg(G.SPMD, G.PL_STACK, 1, 256, flags=G.F_HISTORY),
    "native_history": G.cfg(G.NATIVE, G.PL_STACK, 1, 256, flags=G.F_HISTORY),
    "spmd_sorted": G.cfg(G.SPMD, G.PL_STACK, 1, 256),
    "spmd128_sorted": G.cfg(G.SPMD, G.PL_STACK, 1, 128),
    "spmd_plain_sorted": G.cfg(G.SPMD, G.PL_STACK, 1, 256, flags=G.F_PLAIN),
    "native_sorted": G.cfg(G.NATIVE, G.PL_STACK, 1, 256),
    "csm_sorted": G.cfg(G.CSM, G.PL_STACK, 1, 256),
    "generic_sorted": G.cfg(G.GENERIC, G.PL_STACK, 1, 256),
}

ap = argparse.ArgumentParser()
ap.add_argument("variants", nargs="+")
ap.add_argument("--n", type=int, default=17_000_000)
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--niso", type=int, default=355)
ap.add_argument("--time", action="store_true")
ap.add_argument("--persist", type=float, default=0.0, help="L2 persisting window over the grid, hit ratio")
ap.add_argument("--persist-mb", type=int, default=96)
ap.add_argument("--bins", type=int, default=21, help="log2 union bins; -1: full-range union search")
a = ap.parse_args()
ctx = G.gtr_ctx_create(0)
xs = XsDevice(ctx, X.make_tables(a.niso), union_bins_log2=None if a.bins < 0 else a.bins)
out = torch.zeros(18, dtype=torch.uint64, device="cuda")
if a.persist > 0:
    G.gtr_l2_persist(ctx, xs.grid, xs.grid.numel() * 8, a.persist_mb << 20, a.persist)
    print("persist window", a.persist, a.persist_mb, "MB")
ws = None
for v in a.variants:
    c = VARIANTS[v]
    out.zero_()
    if v.endswith("_sorted"):
        if ws is None:
            ws = torch.empty(G.gtr_xs_sorted_workspace_bytes(a.n), dtype=torch.uint8, device="cuda")
        run = lambda: G.gtr_xs_lookup_sorted(ctx, c, xs.tables, 0, a.n, X.SEED_L, out, ws)  # noqa: E731
    else:
        run = lambda: G.gtr_xs_lookup(ctx, c, xs.tables, 0, a.n, X.SEED_L, out)  # noqa: E731
    run()
    if a.time:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.reps):
            out.zero_()
            run()
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.reps
        qc = G.gtr_launch_cfg(c.num_teams, c.thread_limit, c.mode, c.placement, c.fold, c.smem_stack_bytes,
                              c.flags | (G.F_SORTED if v.endswith("_sorted") else 0))
        info = G.gtr_query_variant(G.K_XS, qc)
        print(f"{v:16s} {ms:8.3f} ms  {a.n / ms / 1e3:8.1f} M lookups/s  regs {info['regs']} "
              f"teams/SM {info['teams_per_sm']}  hash {int(out.cpu()[0])}", flush=True)
    G.gtr_ctx_check(ctx)

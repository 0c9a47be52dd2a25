"""Launch / time the RSBench lookup per variant (ncu captures and A/B timing).

    python tools/rs_launch.py spmd native ... [--n 200000] [--reps 1] [--time]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import gtr_inputs.rs as RS  # noqa: E402
import gtr_inputs.xs as X  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200 import gtr as G  # noqa: E402
from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice  # noqa: E402

VARIANTS = {
    "native": G.cfg(G.NATIVE, G.PL_STACK, 1, 128),
    "native_bucketed": G.cfg(G.NATIVE, G.PL_STACK, 1, 128, flags=G.F_NATIVE_BUCKETED),
    "spmd": G.cfg(G.SPMD, G.PL_STACK, 1, 128),
    "spmd_plain": G.cfg(G.SPMD, G.PL_STACK, 1, 128, flags=G.F_PLAIN),
    "csm": G.cfg(G.CSM, G.PL_STACK, 1, 128),
    "generic": G.cfg(G.GENERIC, G.PL_STACK, 1, 128),
}

ap = argparse.ArgumentParser()
ap.add_argument("variants", nargs="+")
ap.add_argument("--n", type=int, default=200_000)
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--time", action="store_true")
ap.add_argument("--narrow", action="store_true", help="RSBench's 72-byte pole records")
a = ap.parse_args()
ctx = G.gtr_ctx_create(0)
rs = RsDevice(RS.make_tables(), ctx=ctx, wide_poles=not a.narrow)
out = torch.zeros(18, dtype=torch.uint64, device="cuda")
for v in a.variants:
    c = VARIANTS[v]
    out.zero_()
    G.gtr_rs_lookup(ctx, c, rs.tables, 0, a.n, X.SEED_L, out)
    if a.time:
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(a.reps):
            out.zero_()
            G.gtr_rs_lookup(ctx, c, rs.tables, 0, a.n, X.SEED_L, out)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / a.reps
        print(f"{v}: {ms:.3f} ms  {a.n / ms / 1e3:.1f} M lookups/s  hash {int(out[0])}", flush=True)
G.gtr_ctx_check(ctx)
torch.cuda.synchronize()

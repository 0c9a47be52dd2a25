"""Launch the XS-large lookup once per requested variant (for ncu captures).

    python tools/xs_launch.py spmd native csm generic [--n 17000000] [--reps 2]
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
    "spmd": G.cfg(G.SPMD, G.PL_STACK, 1, 256),
    "spmd_runtime": G.cfg(G.SPMD, G.PL_RUNTIME, 0, 256),
    "csm": G.cfg(G.CSM, G.PL_STACK, 1, 256),
    "generic": G.cfg(G.GENERIC, G.PL_STACK, 1, 256),
}

ap = argparse.ArgumentParser()
ap.add_argument("variants", nargs="+")
ap.add_argument("--n", type=int, default=17_000_000)
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--niso", type=int, default=355)
a = ap.parse_args()
ctx = G.gtr_ctx_create(0)
xs = XsDevice(ctx, X.make_tables(a.niso))
out = torch.zeros(18, dtype=torch.uint64, device="cuda")
for v in a.variants:
    for _ in range(a.reps):
        out.zero_()
        G.gtr_xs_lookup(ctx, VARIANTS[v], xs.tables, 0, a.n, X.SEED_L, out)
    G.gtr_ctx_check(ctx)
    print(v, int(out.cpu()[0]))

"""Writes tests/golden/rs_large_10M.json: the oracle's result (hash + 12
material tallies + 4 argmax tallies) over the full RS config 4 workload --
355 nuclides, lookups [0, 10M), SEED_L -- plus the smallest tie margin of the
run (SURVEY PIN-12).  Calls only oracle/ and gtr_inputs/ (the stored value is
the oracle's, never the CUDA path's).  ~8 min on 8 cores.

    python tools/gen_rs_golden.py [--n 10000000] [--threads N]
"""
import argparse
import json
import os
import platform
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
import gtr_inputs.rs as RS  # noqa: E402
import gtr_inputs.xs as X  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--n", type=int, default=10_000_000)
    ap.add_argument("--threads", type=int, default=os.cpu_count() or 8)
    ap.add_argument("--out", default=os.path.join(ROOT, "tests", "golden", "rs_large_10M.json"))
    a = ap.parse_args()
    t = RS.make_tables()
    P = oracle.RsProblem(t)
    t0 = time.time()
    out, _, margin = P.run(0, a.n, X.SEED_L, a.threads)
    dt = time.time() - t0
    rec = {"what": "oracle orc_rs_run over RS config 4 (355 nuclides, ~1000 poles / 100 windows), "
                   "lookups [0, n), seed SEED_L; out = [hash, mat_tally[12], argmax_tally[4], 0]",
           "n": a.n, "seed": X.SEED_L, "out": [int(x) for x in out], "min_tie_margin": margin,
           "generated_by": "tools/gen_rs_golden.py (oracle/ only)", "threads": a.threads,
           "seconds": round(dt, 1), "host": platform.processor() or platform.machine()}
    with open(a.out, "w") as f:
        json.dump(rec, f, indent=1)
    print(json.dumps(rec))


if __name__ == "__main__":
    main()

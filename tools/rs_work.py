"""Write profiles/rs_work.json: the algorithmic fp64 work of the RSBench
lookups bench.py times ("counted by the instrumented
oracle").  Calls only oracle/ (test infrastructure); bench.py reads the file
and never executes the oracle outside its cpu_baseline leg.

    python tools/rs_work.py [--n 2000000]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--first", type=int, default=0)
    ap.add_argument("--n", type=int, default=2_000_000)
    a = ap.parse_args()
    import oracle
    import gtr_inputs.rs as RS
    import gtr_inputs.xs as X
    P = oracle.RsProblem(RS.make_tables())
    counts, flops, trans = P.work(a.first, a.n, X.SEED_L, os.cpu_count() or 1)
    rec = {"workload": "gtr_inputs.rs.make_tables() defaults (355 nuclides, ~1000 poles / 100 windows), "
                       f"lookups [{a.first}, {a.first + a.n}), seed {X.SEED_L}",
           "first": a.first, "n": a.n, "seed": X.SEED_L,
           "nuclide_visits": int(counts[0]), "poles_abrarov": int(counts[1]), "poles_asymptotic": int(counts[2]),
           "flops": flops, "transcendentals": trans,
           "flop_weights": "oracle/rs.c: per nuclide 36, per pole 35, W Abrarov 367, W asymptotic 50 "
                           "(fp64 add/sub/mul/div/sqrt = 1)"}
    out = os.path.join(ROOT, "profiles", "rs_work.json")
    json.dump(rec, open(out, "w"), indent=1)
    print(json.dumps(rec))


if __name__ == "__main__":
    main()

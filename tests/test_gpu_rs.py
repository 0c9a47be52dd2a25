"""GPU parity: RS multipole lookup (config 4) vs the oracle.  sin/cos/atan
differ between glibc and CUDA's libm by about an ulp, so macroscopic XS are
compared within 1e-12 relative per element (sigma_T, sigma_A, sigma_F; sigma_E
= sigma_T - sigma_A cancels, so its bound is relative to its operands,
DESIGN.md R-RS-tol); tallies/hash are exact, guarded by the oracle's
tie-margin audit.  Edge cases: the asymptotic Faddeeva
branch, poles whose |Z|^2 straddles 36 by a few ulps (the branch boundary),
E = 1.0 (window clamp), several chunks per team, the full 10M-lookup run."""
import json
import os
import itertools

import numpy as np
import pytest
import torch

import gtr_inputs.rs as RS
import gtr_inputs.xs as X
from gpu_common import G, ctx, pool, RUNTIME_MODES, PLACEMENTS  # noqa: F401

pytestmark = pytest.mark.gpu


# bucketed chunk = 32 lookups per thread x thread_limit 128 = 4096 lookups;
# 3 chunks + a ragged tail, over 2 teams: every team runs several chunks
# (per-chunk resets, distribute_static, multi-team flush)
N_RS = 3 * 4096 + 77
TEAMS_RS = 2


@pytest.fixture(scope="module")
def rs(orc):
    t = RS.make_tables()
    P = orc.RsProblem(t)
    n = N_RS
    out, v, margin = P.run(1000, n, X.SEED_L, os.cpu_count() or 8, verify=True)
    assert margin > 1e-10, margin        # no argmax can flip under 1e-12 noise
    return t, P, out, v, n


@pytest.fixture(scope="module")
def dev(rs):
    from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice
    return RsDevice(rs[0])


def _check(G, ctx, dev, rs, cfg):
    t, P, o_out, o_v, n = rs
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    v, bufs = dev.verify_buffers(n)
    G.gtr_rs_lookup(ctx, cfg, dev.tables, 1000, n, X.SEED_L, out, v)
    G.gtr_ctx_check(ctx)
    assert np.array_equal(out.cpu().numpy(), o_out)
    assert np.array_equal(bufs["mat"].cpu().numpy(), o_v["mat"])
    assert np.array_equal(bufs["am"].cpu().numpy(), o_v["am"])
    assert_macro_close(bufs["macro"].cpu().numpy(), o_v["macro"])


RTOL = 1e-12


def assert_macro_close(got, want):
    """R-RS-tol: sigma_T, sigma_A, sigma_F within 1e-12 relative, element by
    element; sigma_E = sigma_T - sigma_A within 1e-12 of max(|sigma_T|, |sigma_A|)
    (its operands: the subtraction cancels, its own relative error need not)."""
    err = np.abs(got - want)
    rel = err[:, :3] / np.abs(want[:, :3])
    assert (err[:, :3] <= RTOL * np.abs(want[:, :3])).all(), ("T/A/F", np.nanmax(rel, axis=0))
    opnd = np.maximum(np.abs(want[:, 0]), np.abs(want[:, 1]))
    assert (err[:, 3] <= RTOL * opnd).all(), ("E", (err[:, 3] / opnd).max())


@pytest.mark.parametrize("sched", (0, 4), ids=("bucketed", "plain"))
@pytest.mark.parametrize("variant", list(itertools.product(RUNTIME_MODES, PLACEMENTS, (0, 1), (128,))),
                         ids=lambda v: "m%d-p%d-f%d-t%d" % v)
def test_rs_all_variants(G, ctx, dev, rs, variant, sched):
    m, p, f, nt = variant
    _check(G, ctx, dev, rs, G.cfg(m, p, f, nt, num_teams=TEAMS_RS, flags=sched))


@pytest.mark.parametrize("nt", (128, 256))
def test_rs_native(G, ctx, dev, rs, nt):
    _check(G, ctx, dev, rs, G.cfg(G.NATIVE, G.PL_STACK, 1, nt))


@pytest.mark.parametrize("cfg", [(3, 3, 1, 128), (2, 3, 1, 128), (0, 0, 0, 128)], ids=lambda v: "m%d-p%d-f%d-t%d" % v)
def test_rs_default_teams(G, ctx, dev, rs, cfg):
    """the same lookups over the default one-wave league (many teams, one partial chunk each)"""
    m, p, f, nt = cfg
    _check(G, ctx, dev, rs, G.cfg(m, p, f, nt))


@pytest.fixture(scope="module")
def dev_narrow(rs):
    """RSBench's 72-byte pole records (no wide-pole table)."""
    from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice
    return RsDevice(rs[0], wide_poles=False)


def test_rs_wide_poles_builder(orc, dev, rs):
    """poles_wide[r] = the 72-byte record's 9 words + the pole's lookup-
    invariant factors of exp(12 i Z): word 9 = fast_exp(-12 Z.i) with Z.i =
    -EA.i/2 -- bit-identical to the oracle's orc_fast_exp of the same
    argument -- and words 10, 11 = cos, sin(6 EA.r) (CUDA libm vs numpy:
    within 2 ulp)."""
    t = rs[0]
    raw = np.ascontiguousarray(t["poles"]).view(np.float64).reshape(-1, 9)
    got = dev.poles_wide.cpu().numpy()
    assert np.array_equal(got[:, :9].view(np.uint64), raw.view(np.uint64))
    ea_r, ea_i = raw[:, 0], raw[:, 1]
    idx = np.random.default_rng(0).integers(0, len(raw), 2000)
    for r in idx:
        zi = (0.0 - ea_i[r]) * 0.5
        assert got[r, 9] == orc.fast_exp(-12.0 * zi)
    np.testing.assert_allclose(got[:, 10], np.cos(6.0 * ea_r), rtol=0, atol=5e-16)
    np.testing.assert_allclose(got[:, 11], np.sin(6.0 * ea_r), rtol=0, atol=5e-16)


@pytest.mark.parametrize("cfg", [(0, 0, 0, 128), (2, 3, 1, 128), (3, 3, 1, 128), (3, 0, 0, 128), (4, 3, 1, 128),
                                 (4, 3, 1, 256)], ids=lambda v: "m%d-p%d-f%d-t%d" % v)
def test_rs_narrow_records(G, ctx, dev_narrow, rs, cfg):
    m, p, f, nt = cfg
    _check(G, ctx, dev_narrow, rs, G.cfg(m, p, f, nt))


def test_rs_wide_poles_misaligned_rejected(G, ctx, dev, rs):
    import ctypes
    t = G.gtr_rs_tables.from_buffer_copy(dev.tables)
    t.poles_wide = dev.poles_wide.data_ptr() + 8
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    with pytest.raises(G.GtrError):
        G.gtr_rs_lookup(ctx, G.cfg(G.SPMD, G.PL_STACK, 1, 128), t, 0, 10, X.SEED_L, out)
    assert ctypes.sizeof(t) == ctypes.sizeof(dev.tables)


@pytest.mark.slow
def test_rs_full_size_bench_launch(G, ctx, orc):
    """Config 4 at full size (355 nuclides, 10M lookups) in the launch
    configuration bench.py times (SPMD + heap-to-stack + folding, thread
    limit 128, wide pole records): hash and all 16 tallies of the whole run
    equal the oracle's (tests/golden/rs_large_10M.json, written by
    tools/gen_rs_golden.py from oracle/ alone), and five ranges of 3000
    lookups spread over [0, 10M) match the oracle element by element
    (R-RS-tol) with identical materials and argmaxes."""
    from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice
    with open(os.path.join(os.path.dirname(__file__), "golden", "rs_large_10M.json")) as f:
        gold = json.load(f)
    t = RS.make_tables()
    dev = RsDevice(t, ctx=ctx)
    n = 10_000_000
    assert gold["n"] == n and gold["seed"] == X.SEED_L
    assert gold["min_tie_margin"] > 1e-10         # a 1e-12 perturbation cannot flip any argmax
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    v, bufs = dev.verify_buffers(n)
    G.gtr_rs_lookup(ctx, G.cfg(G.SPMD, G.PL_STACK, 1, 128), dev.tables, 0, n, X.SEED_L, out, v)
    G.gtr_ctx_check(ctx)
    res = out.cpu().numpy()
    assert [int(x) for x in res] == gold["out"]
    P = orc.RsProblem(t)
    m = 3000
    for first in (0, 2_345_678, 5_000_000, 7_777_777, n - m):
        o_out, o_v, margin = P.run(first, m, X.SEED_L, os.cpu_count() or 8, verify=True)
        assert margin > 1e-10
        sl = slice(first, first + m)
        assert np.array_equal(bufs["mat"][sl].cpu().numpy(), o_v["mat"])
        assert np.array_equal(bufs["am"][sl].cpu().numpy(), o_v["am"])
        assert_macro_close(bufs["macro"][sl].cpu().numpy(), o_v["macro"])
    # the other runtime modes of the bench ladder over the whole run: same hash and tallies
    for cfg in (G.cfg(G.CSM, G.PL_STACK, 1, 128), G.cfg(G.NATIVE, G.PL_STACK, 1, 128)):
        out.zero_()
        G.gtr_rs_lookup(ctx, cfg, dev.tables, 0, n, X.SEED_L, out)
        G.gtr_ctx_check(ctx)
        assert [int(x) for x in out.cpu().numpy()] == gold["out"]


# ---------------------------------------------------------------- edge cases
EDGE_CFGS = [(3, 3, 1, 128, 0), (3, 0, 0, 128, 0), (2, 3, 1, 128, 0), (0, 2, 0, 128, 0), (1, 4, 0, 128, 0),
             (3, 3, 1, 128, 4), (4, 3, 1, 128, 0), (4, 3, 1, 256, 0), (4, 3, 1, 128, 32)]


def _edge_run(G, ctx, orc, t, first, n, seed, cfgs=EDGE_CFGS, wide=(True, False)):
    from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice
    P = orc.RsProblem(t)
    o_out, o_v, margin = P.run(first, n, seed, os.cpu_count() or 8, verify=True)
    assert margin > 1e-10, margin
    for w in wide:
        dev = RsDevice(t, ctx=ctx, wide_poles=w)
        for m, p, f, nt, fl in cfgs:
            out = torch.zeros(18, dtype=torch.uint64, device="cuda")
            v, bufs = dev.verify_buffers(n)
            G.gtr_rs_lookup(ctx, G.cfg(m, p, f, nt, num_teams=3, flags=fl), dev.tables, first, n, seed, out, v)
            G.gtr_ctx_check(ctx)
            assert np.array_equal(out.cpu().numpy(), o_out), (w, m, p, f, nt, fl)
            assert np.array_equal(bufs["mat"].cpu().numpy(), o_v["mat"])
            assert np.array_equal(bufs["am"].cpu().numpy(), o_v["am"])
            assert_macro_close(bufs["macro"].cpu().numpy(), o_v["macro"])
    return P


def _copy(t):
    return {k: (v.copy() if isinstance(v, np.ndarray) else v) for k, v in t.items()}


def test_rs_asymptotic_branch(G, ctx, orc):
    """Poles far from the sampled energies: EA.i in {-13, -20} (Z.i = 6.5, 10)
    and |EA.r - E| >= 12, so |Z| >= 6 takes the 2-pole asymptotic W; the rest
    keep the workload's EA in [0,1)^2 (the Abrarov series).  Both branches are
    compared with the oracle per lookup."""
    t = _copy(RS.make_tables(avg_poles=60, avg_windows=6, seed=77))
    rng = np.random.default_rng(12)
    EA = t["poles"]["EA"]
    sel = rng.random(EA.shape[:2])
    EA[..., 1] = np.where(sel < 0.2, -13.0, np.where(sel < 0.4, -20.0, EA[..., 1]))
    shift = np.where(rng.random(EA.shape[:2]) < 0.5, -1.0, 1.0) * (12.5 + 30.0 * rng.random(EA.shape[:2]))
    EA[..., 0] = np.where((sel >= 0.4) & (sel < 0.7), EA[..., 0] + shift, EA[..., 0])
    P = _edge_run(G, ctx, orc, t, 0, 6000, X.SEED_L)
    counts, _, _ = P.work(0, 6000, X.SEED_L, os.cpu_count() or 8)
    assert counts[2] > 0.5 * counts[1] > 0                 # both branches well populated


def test_rs_branch_boundary(G, ctx, orc):
    """Poles constructed per lookup so that |Z|^2 = Z.r^2 + Z.i^2 (each op
    rounded, as the oracle computes it before its sqrt) is within 4 ulps of 36
    on both sides, 36 exactly included: the GPU must take the same Faddeeva
    branch as the oracle's sqrt(|Z|^2) < 6 (an FMA-contracted or reassociated
    predicate would flip some).  Z.i in (-0.5, 0] as in the workload."""
    base = RS.make_tables(avg_poles=8, avg_windows=1, seed=91)
    t = _copy(base)
    L, first, seed = 256, 5, X.SEED_L
    n_nuc = int(t["n_nuc"])
    per_nuc = [[] for _ in range(n_nuc)]
    u36 = np.spacing(np.float64(36.0))
    rng = np.random.default_rng(8)
    hits = {}
    for i in range(first, first + L):
        E, s = orc.lcg_double(orc.lcg_ff(seed, 2 * i))
        mat, _ = orc.pick_mat(s)
        nn = int(t["num_nucs"][mat])
        nuc = int(t["mats"][mat, i % nn])
        found = 0
        for _ in range(4000):
            b = np.float64(rng.uniform(0.0, 0.49))               # Z.i = -b
            sgn = 1.0 if rng.random() < 0.5 else -1.0
            a0 = sgn * np.sqrt(np.float64(36.0) - b * b)
            ear = np.float64(E) - np.float64(2.0) * a0
            for k in range(-3, 4):
                er = ear
                for _ in range(abs(k)):
                    er = np.nextafter(er, np.inf if k > 0 else -np.inf)
                zr = (np.float64(E) - er) * np.float64(0.5) - (np.float64(0.0) - np.float64(2.0) * b) * 0.0
                zi = np.float64(-b)
                x = zr * zr + zi * zi
                d = int(round((x - 36.0) / u36))
                if abs(d) <= 4 and len(per_nuc[nuc]) < 64:
                    per_nuc[nuc].append((er, 2.0 * b, d))
                    hits[d] = hits.get(d, 0) + 1
                    found += 1
            if found >= 6:
                break
    assert all(hits.get(d, 0) > 0 for d in (-2, -1, 0, 1)), hits
    max_p = max(8, max(len(p) for p in per_nuc))
    poles = np.zeros((n_nuc, max_p), dtype=RS.POLE_DTYPE)
    rr = np.random.default_rng(9)
    for n in range(n_nuc):
        for j, (er, ei, _) in enumerate(per_nuc[n]):
            poles[n, j]["EA"] = (er, ei)
            poles[n, j]["RT"] = rr.random(2)
            poles[n, j]["RA"] = rr.random(2)
            poles[n, j]["RF"] = rr.random(2)
            poles[n, j]["l_value"] = rr.integers(0, 4)
    t["poles"] = poles
    t["max_poles"] = max_p
    t["n_poles"] = np.array([len(p) for p in per_nuc], dtype=np.int32)
    t["n_windows"][:] = 1
    w = np.zeros((n_nuc, 1), dtype=RS.WIN_DTYPE)
    w["T"], w["A"], w["F"] = base["windows"]["T"][:, :1], base["windows"]["A"][:, :1], base["windows"]["F"][:, :1]
    w["start"] = 0
    w["end"] = t["n_poles"][:, None]                        # every pole of the nuclide
    t["windows"] = w
    t["max_windows"] = 1
    P = _edge_run(G, ctx, orc, t, first, L, seed)
    counts, _, _ = P.work(first, L, seed)
    assert counts[1] > 0 and counts[2] > 0


def test_rs_energy_exactly_one(G, ctx, orc):
    """A seed whose first draw is 2^63 - 1: E = 1.0 exactly, so the window
    index E / (1/n_windows) = n_windows is clamped to the last window
    (c4 step 1); 64 lookups of that seed vs the oracle."""
    a, M = 2806196910506780709, 1 << 63
    seed = (pow(a, -1, M) * ((M - 1) - 1)) % M
    E, _ = orc.lcg_double(seed)
    assert E == 1.0
    t = RS.make_tables(avg_poles=100, avg_windows=10, seed=5)
    _edge_run(G, ctx, orc, t, 0, 64, seed)


def test_rs_native_bucketed(G, ctx, dev, dev_narrow, rs):
    """GTR_F_NATIVE_BUCKETED: the bucketed schedule as plain CUDA -- same
    lookups (R-RS-tol), several chunks per team and the default league."""
    for d in (dev, dev_narrow):
        _check(G, ctx, d, rs, G.cfg(G.NATIVE, G.PL_STACK, 1, 128, flags=G.F_NATIVE_BUCKETED))
        _check(G, ctx, d, rs, G.cfg(G.NATIVE, G.PL_STACK, 1, 128, num_teams=TEAMS_RS, flags=G.F_NATIVE_BUCKETED))

"""GPU parity: RS multipole lookup (config 4) vs the oracle.  sin/cos/atan
differ between glibc and CUDA's libm by about an ulp, so macroscopic XS are
compared within 1e-12 relative; tallies/hash are exact, guarded by the
oracle's tie-margin audit."""
import itertools

import numpy as np
import pytest
import torch

import gtr_inputs.rs as RS
import gtr_inputs.xs as X
from gpu_common import G, ctx, pool, RUNTIME_MODES, PLACEMENTS  # noqa: F401

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def rs(orc):
    t = RS.make_tables()
    P = orc.RsProblem(t)
    n = 4000
    out, v, margin = P.run(1000, n, X.SEED_L, 8, verify=True)
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
    # 1e-12 relative to the lookup's largest channel: sigE = sigT - sigA can
    # cancel, so its error is bounded relative to the operands, not the result
    got, want = bufs["macro"].cpu().numpy(), o_v["macro"]
    scale = np.abs(want).max(axis=1, keepdims=True)
    assert (np.abs(got - want) <= 1e-12 * scale).all(), np.abs(got - want).max()


@pytest.mark.parametrize("sched", (0, 4), ids=("bucketed", "plain"))
@pytest.mark.parametrize("variant", list(itertools.product(RUNTIME_MODES, PLACEMENTS, (0, 1), (128,))),
                         ids=lambda v: "m%d-p%d-f%d-t%d" % v)
def test_rs_all_variants(G, ctx, dev, rs, variant, sched):
    m, p, f, nt = variant
    _check(G, ctx, dev, rs, G.cfg(m, p, f, nt, flags=sched))


@pytest.mark.parametrize("nt", (128, 256))
def test_rs_native(G, ctx, dev, rs, nt):
    _check(G, ctx, dev, rs, G.cfg(G.NATIVE, G.PL_STACK, 1, nt))


@pytest.fixture(scope="module")
def dev_narrow(rs):
    """RSBench's 72-byte pole records (no wide-pole table)."""
    from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice
    return RsDevice(rs[0], wide_poles=False)


def test_rs_wide_poles_builder(dev, rs):
    """poles_wide[r] = the 72-byte record's 9 words + 3 zero words."""
    t = rs[0]
    raw = np.ascontiguousarray(t["poles"]).view(np.float64).reshape(-1, 9)
    got = dev.poles_wide.cpu().numpy()
    assert np.array_equal(got[:, :9].view(np.uint64), raw.view(np.uint64))
    assert (got[:, 9:] == 0).all()


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
    limit 128, wide pole records): the whole run's tallies are consistent
    (every lookup counted once, hash = sum (argmax+1) x tally), and five
    ranges of 3000 lookups spread over [0, 10M) match the oracle element by
    element (R-RS-tol) with identical materials and argmaxes."""
    import os
    from paper_conf_cgo_hubercgtddcd22_b200.problems import RsDevice
    t = RS.make_tables()
    dev = RsDevice(t, ctx=ctx)
    n = 10_000_000
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    v, bufs = dev.verify_buffers(n)
    G.gtr_rs_lookup(ctx, G.cfg(G.SPMD, G.PL_STACK, 1, 128), dev.tables, 0, n, X.SEED_L, out, v)
    G.gtr_ctx_check(ctx)
    res = out.cpu().numpy()
    assert int(res[1:13].sum()) == n and int(res[13:17].sum()) == n
    assert int(res[0]) == sum((k + 1) * int(res[13 + k]) for k in range(4))
    P = orc.RsProblem(t)
    m = 3000
    for first in (0, 2_345_678, 5_000_000, 7_777_777, n - m):
        o_out, o_v, margin = P.run(first, m, X.SEED_L, os.cpu_count() or 8, verify=True)
        assert margin > 1e-10
        sl = slice(first, first + m)
        assert np.array_equal(bufs["mat"][sl].cpu().numpy(), o_v["mat"])
        assert np.array_equal(bufs["am"][sl].cpu().numpy(), o_v["am"])
        got, want = bufs["macro"][sl].cpu().numpy(), o_v["macro"]
        scale = np.abs(want).max(axis=1, keepdims=True)
        assert (np.abs(got - want) <= 1e-12 * scale).all(), (first, np.abs(got - want).max())

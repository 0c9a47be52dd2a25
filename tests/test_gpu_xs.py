"""GPU parity: XS lookup (configs 1 and 5) through libgtr.so vs the oracle.

Bar (BASELINE.json north_star): hash, tallies and every integer index
bit-exact; fp64 macroscopic cross sections within 1e-12 relative -- here they
are bit-identical, because both sides round every operation separately
(AMB-12), and the test asserts that.  Results identical across all modes,
placements and folds.
"""
import numpy as np
import pytest
import torch

import gtr_inputs.xs as X
from gpu_common import G, ctx, pool, all_variants, vid  # noqa: F401

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def small(orc):
    t = X.make_tables(68)
    P = orc.XsProblem(t)
    n = 100000
    out, v = P.run(0, n, X.SEED_L, 4, verify=True)
    return t, P, out, v, n


@pytest.fixture(scope="module")
def dev_small(G, ctx, small):
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    return XsDevice(ctx, small[0])


def test_unionized_grid_matches_oracle(dev_small, small):
    t, P, *_ = small
    assert np.array_equal(dev_small.egrid.cpu().numpy(), P.egrid)
    assert np.array_equal(dev_small.index_grid.cpu().numpy(), P.index_grid)


def test_union_bins_builder(G, ctx, dev_small, small):
    """bins[b] = searchsorted(egrid, b / 2^L, 'left') on the oracle's egrid."""
    t, P, *_ = small
    L = dev_small.union_bins_log2
    want = np.searchsorted(P.egrid, np.arange((1 << L) + 1) / float(1 << L), side="left")
    assert np.array_equal(dev_small.union_bins.cpu().numpy().astype(np.int64), want)


@pytest.fixture(scope="module")
def dev_small_plain(G, ctx, small):
    """Tables without the union bins: the full-range binary search."""
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    return XsDevice(ctx, small[0], union_bins_log2=None)


@pytest.mark.parametrize("sched", (0, 4), ids=("bucketed", "plain"))
@pytest.mark.parametrize("variant", [(m, p, f, nt) for m in (0, 1, 2, 3) for p, f in ((3, 1), (0, 0))
                                     for nt in (128, 256)], ids=vid)
def test_plain_tables_bit_exact(G, ctx, dev_small_plain, small, variant, sched):
    t, P, o_out, o_v, n = small
    m, p, f, nt = variant
    out, v = _run(G, ctx, dev_small_plain, G.cfg(m, p, f, nt, flags=sched), 0, n)
    _assert_same(out, v, o_out, o_v)
    out, v = _run(G, ctx, dev_small_plain, G.cfg(G.NATIVE, G.PL_STACK, 1, nt), 0, n)
    _assert_same(out, v, o_out, o_v)


@pytest.mark.parametrize("log2b", (0, 1, 7, 26))
def test_union_bins_extreme_sizes(G, ctx, small, log2b):
    """One bin (the full range), a few, and 2^26 bins (mostly empty, every
    non-empty bin holds one energy): same results."""
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    t, P, o_out, o_v, n = small
    dev = XsDevice(ctx, t, union_bins_log2=log2b)
    for mode in (G.SPMD, G.NATIVE):
        out, v = _run(G, ctx, dev, G.cfg(mode, G.PL_STACK, 1, 256), 0, 20000)
        _assert_same(out, v, *P.run(0, 20000, X.SEED_L, 4, verify=True))


@pytest.mark.parametrize("log2b", (None, 0, 3, 21))
def test_energies_outside_the_grid(G, ctx, orc, log2b):
    """Gridpoint energies squeezed into [0.25, 0.75): lookups with E below the
    first union energy (u = 0) and above the last (u = n_union - 2, the
    clamp), through every search path."""
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    t = X.make_tables(68, 2000)
    t["grid"][:, :, 0] = 0.25 + 0.5 * t["grid"][:, :, 0]
    P = orc.XsProblem(t)
    n = 30000
    o_out, o_v = P.run(0, n, X.SEED_L, 4, verify=True)
    assert (o_v["u"] == 0).sum() > 1000 and (o_v["u"] == P.n_union - 2).sum() > 1000
    dev = XsDevice(ctx, t, union_bins_log2=log2b)
    for c in (G.cfg(G.SPMD, G.PL_STACK, 1, 256), G.cfg(G.NATIVE, G.PL_STACK, 1, 256),
              G.cfg(G.GENERIC, G.PL_RUNTIME, 0, 128), G.cfg(G.CSM, G.PL_STACK, 1, 128, flags=G.F_PLAIN)):
        out, v = _run(G, ctx, dev, c, 0, n)
        _assert_same(out, v, o_out, o_v)


def test_energy_exactly_one(G, ctx, dev_small, dev_small_plain, small):
    """A lookup seed whose first draw is 2^63 - 1: u64 -> f64 rounds it to
    2^63, so E = 1.0 exactly (c1.1) -- the top edge of the last union bin.
    Lookups 0..63 of that seed through both search paths vs the oracle."""
    t, P, *_ = small
    a, M = 2806196910506780709, 1 << 63
    a_inv = pow(a, -1, M)
    seed = (a_inv * ((M - 1) - 1)) % M            # a * seed + 1 = 2^63 - 1
    o_out, o_v = P.run(0, 64, seed, 1, verify=True)
    assert o_v["u"][0] == P.n_union - 2          # E = 1.0 is above every energy
    for dev in (dev_small, dev_small_plain):
        for c in (G.cfg(G.SPMD, G.PL_STACK, 1, 256), G.cfg(G.NATIVE, G.PL_STACK, 1, 256),
                  G.cfg(G.CSM, G.PL_STACK, 1, 128, flags=G.F_PLAIN)):
            out = torch.zeros(18, dtype=torch.uint64, device="cuda")
            v, bufs = dev.verify_buffers(64)
            G.gtr_xs_lookup(ctx, c, dev.tables, 0, 64, seed, out, v)
            G.gtr_ctx_check(ctx)
            _assert_same(out.cpu().numpy(), {k: b.cpu().numpy() for k, b in bufs.items()}, o_out, o_v)


def _seed_e_one():
    a, M = 2806196910506780709, 1 << 63
    return (pow(a, -1, M) * ((M - 1) - 1)) % M     # a * seed + 1 = 2^63 - 1


def test_energy_exactly_one_grid_types_and_sorted(G, ctx, dev_grid, dev_small, small):
    """E = 1.0 through the nuclide grid, the hash grid (bin E / du = hash_bins
    clamped to the last bin, DESIGN.md R-XS-hash1 -- unclamped it read one row
    past the hash table) and the sorted event mode (sort key clamped to the
    last energy bucket): bit-identical to the oracle's unionized lookups."""
    gt, dev = dev_grid
    t, P, *_ = small
    seed = _seed_e_one()
    o_out, o_v = P.run(0, 64, seed, 1, verify=True)
    cfgs = (G.cfg(G.SPMD, G.PL_STACK, 1, 256), G.cfg(G.NATIVE, G.PL_STACK, 1, 256),
            G.cfg(G.CSM, G.PL_STACK, 1, 128, flags=G.F_PLAIN), G.cfg(G.GENERIC, G.PL_RUNTIME, 0, 128))
    for c in cfgs:
        out = torch.zeros(18, dtype=torch.uint64, device="cuda")
        v, bufs = dev.verify_buffers(64)
        G.gtr_xs_lookup(ctx, c, dev.tables, 0, 64, seed, out, v)
        G.gtr_ctx_check(ctx)
        assert np.array_equal(out.cpu().numpy(), o_out)
        assert np.array_equal(bufs["macro"].cpu().numpy().view(np.uint64), o_v["macro"].view(np.uint64))
        assert np.array_equal(bufs["mat"].cpu().numpy(), o_v["mat"])
    for d in (dev, dev_small):
        for c in cfgs[:2]:
            out = torch.zeros(18, dtype=torch.uint64, device="cuda")
            v, bufs = d.verify_buffers(64)
            ws = torch.empty(G.gtr_xs_sorted_workspace_bytes(64), dtype=torch.uint8, device="cuda")
            G.gtr_xs_lookup_sorted(ctx, c, d.tables, 0, 64, seed, out, ws, v)
            G.gtr_ctx_check(ctx)
            assert np.array_equal(out.cpu().numpy(), o_out)
            assert np.array_equal(bufs["macro"].cpu().numpy().view(np.uint64), o_v["macro"].view(np.uint64))


def _run(G, ctx, dev, cfg, first, n, verify=True):
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    v, bufs = dev.verify_buffers(n) if verify else (None, None)
    G.gtr_xs_lookup(ctx, cfg, dev.tables, first, n, X.SEED_L, out, v)
    G.gtr_ctx_check(ctx)
    return out.cpu().numpy(), ({k: b.cpu().numpy() for k, b in bufs.items()} if verify else None)


def _assert_same(out, v, o_out, o_v, lo=0, hi=None):
    assert np.array_equal(out, o_out)
    hi = len(o_v["mat"]) if hi is None else hi
    assert np.array_equal(v["mat"], o_v["mat"][lo:hi])
    assert np.array_equal(v["u"].astype(np.uint32), o_v["u"][lo:hi])
    assert np.array_equal(v["am"], o_v["am"][lo:hi])
    # bit-identical fp64 (stronger than the 1e-12 bar)
    assert np.array_equal(v["macro"].view(np.uint64), o_v["macro"][lo:hi].view(np.uint64))


@pytest.mark.parametrize("sched", (0, 4), ids=("bucketed", "plain"))
@pytest.mark.parametrize("variant", all_variants((128, 256)), ids=vid)
def test_all_variants_bit_exact(G, ctx, dev_small, small, variant, sched):
    t, P, o_out, o_v, n = small
    m, p, f, nt = variant
    out, v = _run(G, ctx, dev_small, G.cfg(m, p, f, nt, flags=sched), 0, n)
    _assert_same(out, v, o_out, o_v)


@pytest.mark.parametrize("nt", (128, 256, 512))
def test_native_bit_exact(G, ctx, dev_small, small, nt):
    t, P, o_out, o_v, n = small
    out, v = _run(G, ctx, dev_small, G.cfg(G.NATIVE, G.PL_STACK, 1, nt), 0, n)
    _assert_same(out, v, o_out, o_v)


@pytest.mark.parametrize("mode", (0, 2, 3, 4))
@pytest.mark.parametrize("first,n,teams", [(0, 1, 0), (777, 12345, 0), (99991, 9, 3), (5, 70001, 1)])
def test_ragged_ranges(G, ctx, dev_small, small, orc, mode, first, n, teams):
    t, P, *_ = small
    o_out, o_v = P.run(first, n, X.SEED_L, 4, verify=True)
    out, v = _run(G, ctx, dev_small, G.cfg(mode, G.PL_STACK, 1, 128, num_teams=teams), first, n)
    _assert_same(out, v, o_out, o_v)


def test_empty_request_is_noop(G, ctx, dev_small):
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    G.gtr_xs_lookup(ctx, G.cfg(), dev_small.tables, 0, 0, X.SEED_L, out)
    G.gtr_ctx_check(ctx)
    assert out.cpu().numpy().sum() == 0


def test_host_io_entry_point(G, ctx, dev_small, small):
    t, P, o_out, o_v, n = small
    h_out = torch.zeros(18, dtype=torch.uint64).pin_memory()
    req = G.gtr_xs_request(0, n, X.SEED_L)
    for mode in (G.SPMD, G.NATIVE, G.GENERIC):
        G.gtr_xs_lookup_host(ctx, G.cfg(mode, G.PL_STACK, 1, 256), dev_small.tables, req, h_out)
        assert np.array_equal(h_out.numpy(), o_out)


def test_runtime_stack_overflow_falls_back_to_pool(G, ctx, dev_small, small):
    # 16-byte shared stack: most globalized variables spill to the global pool
    t, P, o_out, o_v, n = small
    for mode in (G.GENERIC, G.SPMD):
        out, v = _run(G, ctx, dev_small, G.cfg(mode, G.PL_RUNTIME, 0, 128, smem_stack_bytes=16), 0, n)
        _assert_same(out, v, o_out, o_v)


def test_fallback_high_water_mark(G, ctx, dev_small, small):
    """gtr_ctx_fallback_high_water: 0 when every globalized variable stays in
    registers / shared memory; with the forced global placement the lookup's
    locals (seed 8 B, macro_xs 40 B, xs 40 B, AMB-7) live in the pool -- at
    least the accumulation region's 80 B at once, and never more than the
    88 B of all three plus the main thread's 16-byte chunk struct."""
    t, P, o_out, o_v, n = small
    G.gtr_ctx_fallback_high_water(ctx, reset=True)
    for m in (G.SPMD, G.CSM):
        _run(G, ctx, dev_small, G.cfg(m, G.PL_STACK, 1, 128), 0, 20000, verify=False)
    assert G.gtr_ctx_fallback_high_water(ctx, reset=True) == 0
    for m in (G.SPMD, G.GENERIC):
        _run(G, ctx, dev_small, G.cfg(m, G.PL_GLOBAL, 0, 128), 0, 20000, verify=False)
        hw = G.gtr_ctx_fallback_high_water(ctx, reset=True)
        assert 80 <= hw <= 104 and hw % 8 == 0, (m, hw)
    # the runtime placement spills past a 16-byte shared stack into the pool
    _run(G, ctx, dev_small, G.cfg(G.SPMD, G.PL_RUNTIME, 0, 128, smem_stack_bytes=16), 0, 20000, verify=False)
    assert G.gtr_ctx_fallback_high_water(ctx, reset=True) > 0
    _run(G, ctx, dev_small, G.cfg(G.SPMD, G.PL_RUNTIME, 0, 128), 0, 20000, verify=False)
    assert G.gtr_ctx_fallback_high_water(ctx) == 0


def test_heap_exhaustion_reports_eheap(G, dev_small):
    # no fallback pool at all: GTR_PL_GLOBAL cannot allocate -> GTR_EHEAP
    c = G.gtr_ctx_create(0, None, 0)
    try:
        out = torch.zeros(18, dtype=torch.uint64, device="cuda")
        G.gtr_xs_lookup(c, G.cfg(G.SPMD, G.PL_GLOBAL, 1, 128), dev_small.tables, 0, 1000, X.SEED_L, out)
        assert G.gtr_ctx_check(c, raise_on_error=False) == G.GTR_EHEAP
        assert G.gtr_ctx_check(c, raise_on_error=False) == G.GTR_OK     # cleared
    finally:
        G.gtr_ctx_destroy(c)


def test_invalid_configs_rejected(G, ctx, dev_small):
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    for bad in (G.cfg(thread_limit=100), G.cfg(mode=7), G.cfg(placement=9), G.cfg(thread_limit=96)):
        with pytest.raises(G.GtrError):
            G.gtr_xs_lookup(ctx, bad, dev_small.tables, 0, 10, X.SEED_L, out)


def test_duplicate_energies_golden(G, ctx):
    """The hand-worked duplicate-energy case (tests/golden/xs_dup_index.txt,
    SURVEY c2.5): union grid and the sequential rule's lagging index grid."""
    import os
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    t = X.make_tables(2, 4)
    t["grid"][0, :, 0] = [0.1, 0.2, 0.2, 0.5]
    t["grid"][1, :, 0] = [0.2, 0.3, 0.6, 0.7]
    golden = np.loadtxt(os.path.join(os.path.dirname(__file__), "golden", "xs_dup_index.txt"), dtype=np.int64)
    dev = XsDevice(ctx, t, union_bins_log2=None)
    assert np.array_equal(dev.egrid.cpu().numpy(), [0.1, 0.2, 0.2, 0.2, 0.3, 0.5, 0.6, 0.7])
    assert np.array_equal(dev.index_grid.cpu().numpy(), golden)


def test_duplicate_energies_sequential_rule(G, ctx, orc):
    """Duplicate gridpoint energies within and across nuclides: the GPU
    builders reproduce the oracle's union grid and its sequential-rule index
    grid (which lags the closed-form count), and every mode's lookups match."""
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    t = X.make_tables(3, 50)
    g = t["grid"]
    g[0, 11, 0] = g[0, 10, 0]                         # a pair within nuclide 0
    g[2, 21, 0] = g[2, 22, 0] = g[2, 20, 0]           # a triple within nuclide 2
    g[1, 30, 0] = g[0, 30, 0]                         # across nuclides
    g[2, 40, 0] = g[0, 40, 0] = g[1, 40, 0]
    for n in range(3):
        g[n] = g[n][np.argsort(g[n, :, 0], kind="stable")]
    P = orc.XsProblem(t)
    closed = np.clip(np.stack([np.searchsorted(g[n, :, 0], P.egrid, side="right") - 1 for n in range(3)], 1),
                     0, g.shape[1] - 2)
    assert (P.index_grid != closed).any()             # the lag is exercised
    for log2b in (None, 8):
        dev = XsDevice(ctx, t, union_bins_log2=log2b)
        assert np.array_equal(dev.egrid.cpu().numpy(), P.egrid)
        assert np.array_equal(dev.index_grid.cpu().numpy(), P.index_grid)
        n = 20000
        o_out, o_v = P.run(0, n, X.SEED_L, 4, verify=True)
        for c in (G.cfg(G.SPMD, G.PL_STACK, 1, 256), G.cfg(G.CSM, G.PL_STACK, 1, 128),
                  G.cfg(G.GENERIC, G.PL_RUNTIME, 0, 128), G.cfg(G.NATIVE, G.PL_STACK, 1, 256),
                  G.cfg(G.SPMD, G.PL_STACK, 1, 256, flags=G.F_PLAIN)):
            _assert_same(*_run(G, ctx, dev, c, 0, n), o_out, o_v)
        _assert_same(*_run_sorted(G, ctx, dev, G.cfg(G.SPMD, G.PL_STACK, 1, 256), 0, n), o_out, o_v)


def test_unsorted_energies_detected(G, ctx):
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    t = X.make_tables(3, 50)
    t["grid"][1, 10, 0], t["grid"][1, 11, 0] = t["grid"][1, 11, 0], t["grid"][1, 10, 0]
    with pytest.raises(G.GtrError):
        XsDevice(ctx, t)


@pytest.fixture(scope="module", params=[1, 2], ids=["nuclide_grid", "hash_grid"])
def dev_grid(request, G, ctx, small):
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    return request.param, XsDevice(ctx, small[0], grid_type=request.param, hash_bins=10000)


def test_hash_grid_builder_matches_oracle(G, ctx, small, orc):
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    t = small[0]
    dev = XsDevice(ctx, t, grid_type=2, hash_bins=997)
    P = orc.XsProblem(t, build_index=False, grid_type=2, hash_bins=997)
    assert np.array_equal(dev.hash_index.cpu().numpy(), P.hash_index)
    assert np.array_equal(dev.energies.cpu().numpy(), t["grid"][:, :, 0])


@pytest.mark.parametrize("variant", [(m, p, f, 256) for m in (0, 1, 2, 3) for p, f in ((3, 1), (0, 0), (4, 0))],
                         ids=vid)
@pytest.mark.parametrize("sched", (0, 4), ids=("bucketed", "plain"))
def test_grid_types_bit_exact(G, ctx, dev_grid, small, variant, sched):
    # the three grid types bracket the same gridpoints: macro XS, argmax and
    # tallies bit-identical to the (oracle-pinned) unionized results
    gt, dev = dev_grid
    t, P, o_out, o_v, n = small
    m, p, f, nt = variant
    out, v = _run(G, ctx, dev, G.cfg(m, p, f, nt, flags=sched), 0, n)
    assert np.array_equal(out, o_out)
    assert np.array_equal(v["mat"], o_v["mat"]) and np.array_equal(v["am"], o_v["am"])
    assert np.array_equal(v["macro"].view(np.uint64), o_v["macro"].view(np.uint64))


def test_grid_types_native(G, ctx, dev_grid, small):
    gt, dev = dev_grid
    t, P, o_out, o_v, n = small
    out, v = _run(G, ctx, dev, G.cfg(G.NATIVE, G.PL_STACK, 1, 256), 0, n)
    assert np.array_equal(out, o_out)
    assert np.array_equal(v["macro"].view(np.uint64), o_v["macro"].view(np.uint64))


# ---------------------------------------------------------------- SURVEY NEXT f2
@pytest.mark.parametrize("variant", all_variants((128, 256)) + [(4, 3, 1, 128), (4, 3, 1, 256)], ids=vid)
def test_history_mode_bit_exact(G, ctx, dev_small, small, variant):
    """XSBench's history-based mode: a thread = a particle of 34 consecutive
    lookups; same sampling, so the same results."""
    t, P, o_out, o_v, n = small
    m, p, f, nt = variant
    out, v = _run(G, ctx, dev_small, G.cfg(m, p, f, nt, flags=G.F_HISTORY), 0, n)
    _assert_same(out, v, o_out, o_v)


def _run_sorted(G, ctx, dev, cfg, first, n):
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    v, bufs = dev.verify_buffers(n)
    ws = torch.empty(G.gtr_xs_sorted_workspace_bytes(n), dtype=torch.uint8, device="cuda")
    G.gtr_xs_lookup_sorted(ctx, cfg, dev.tables, first, n, X.SEED_L, out, ws, v)
    G.gtr_ctx_check(ctx)
    return out.cpu().numpy(), {k: b.cpu().numpy() for k, b in bufs.items()}


@pytest.mark.parametrize("variant", all_variants((256,)) + [(4, 3, 1, 256)], ids=vid)
def test_sorted_mode_bit_exact(G, ctx, dev_small, small, variant):
    """Lookups counting-sorted by (material, energy) before the lookup pass:
    per-lookup records (indexed by lookup) and tallies identical."""
    t, P, o_out, o_v, n = small
    m, p, f, nt = variant
    out, v = _run_sorted(G, ctx, dev_small, G.cfg(m, p, f, nt), 0, n)
    _assert_same(out, v, o_out, o_v)


@pytest.mark.parametrize("first,n", [(0, 1), (31337, 4097), (3, 70001)])
def test_sorted_mode_ragged(G, ctx, dev_small, small, first, n):
    t, P, *_ = small
    o_out, o_v = P.run(first, n, X.SEED_L, 4, verify=True)
    for mode in (G.SPMD, G.GENERIC, G.NATIVE):
        for flags in (0, G.F_PLAIN):                 # staged nuclide loops / whole lookups per thread
            out, v = _run_sorted(G, ctx, dev_small, G.cfg(mode, G.PL_STACK, 1, 128, flags=flags), first, n)
            _assert_same(out, v, o_out, o_v)


def test_sorted_mode_grid_types(G, ctx, dev_grid, small):
    gt, dev = dev_grid
    t, P, o_out, o_v, n = small
    out, v = _run_sorted(G, ctx, dev, G.cfg(G.SPMD, G.PL_STACK, 1, 256), 0, n)
    assert np.array_equal(out, o_out)
    assert np.array_equal(v["macro"].view(np.uint64), o_v["macro"].view(np.uint64))


@pytest.fixture(scope="module")
def dense(G, ctx, orc):
    """68 nuclides x 2000 gridpoints and 300,000 lookups: after the sort a
    warp's 32 lookups mostly share each nuclide's gridpoint pair, so the
    warp-coherent path (CoherentRegion) takes its uniform branch for most
    positions, its two-record branch for the rest and, near the sparse
    materials, the direct gather of a k beyond the staged records."""
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    t = X.make_tables(68, 2000)
    P = orc.XsProblem(t)
    return P, XsDevice(ctx, t)


@pytest.mark.parametrize("cfg", [(3, 3, 1, 256, 0, 0), (3, 0, 0, 256, 0, 0), (3, 3, 1, 128, 3, 0),
                                 (2, 3, 1, 256, 0, 0), (2, 1, 0, 128, 2, 0), (0, 3, 1, 256, 0, 0),
                                 (1, 0, 0, 128, 0, 0), (3, 4, 0, 256, 0, 0), (4, 3, 1, 256, 0, 1),
                                 (4, 3, 1, 128, 5, 1)],
                         ids=lambda c: f"m{c[0]}_p{c[1]}_f{c[2]}_t{c[3]}_teams{c[4]}_nb{c[5]}")
@pytest.mark.parametrize("first,n", [(0, 300000), (12345, 77777)])
def test_sorted_coherent_dense(G, ctx, dense, cfg, first, n):
    P, dev = dense
    m, p, f, nt, teams, nb = cfg
    o_out, o_v = P.run(first, n, X.SEED_L, 8, verify=True)
    c = G.cfg(m, p, f, nt, num_teams=teams, flags=G.F_NATIVE_BUCKETED if nb else 0)
    out, v = _run_sorted(G, ctx, dev, c, first, n)
    _assert_same(out, v, o_out, o_v)


@pytest.mark.parametrize("mode", (0, 2, 3, 4))
def test_sorted_host_and_peers(G, ctx, dev_small, small, mode):
    """The sorted event mode through its host-buffer entry point (request
    copied to the device, results copied back) and with the fused peer
    combine (the same buffer listed 3 times gets 3 x the oracle)."""
    t, P, o_out, o_v, n = small
    c = G.cfg(mode, G.PL_STACK, 1, 256)
    ws = torch.empty(G.gtr_xs_sorted_workspace_bytes(n), dtype=torch.uint8, device="cuda")
    h_out = torch.zeros(18, dtype=torch.uint64).pin_memory()
    G.gtr_xs_lookup_sorted_host(ctx, c, dev_small.tables, G.gtr_xs_request(0, n, X.SEED_L), h_out, ws)
    G.gtr_ctx_check(ctx)
    assert np.array_equal(h_out.numpy(), o_out)
    o2, _ = P.run(777, 5000, X.SEED_L + 9, 4)
    G.gtr_xs_lookup_sorted_host(ctx, c, dev_small.tables, G.gtr_xs_request(777, 5000, X.SEED_L + 9), h_out, ws)
    G.gtr_ctx_check(ctx)
    assert np.array_equal(h_out.numpy(), o2)
    buf = torch.zeros(18, dtype=torch.uint64, device="cuda")
    G.gtr_xs_sort_lookups(ctx, dev_small.tables, 0, n, X.SEED_L, ws)
    G.gtr_xs_lookup_presorted_peers(ctx, c, dev_small.tables, 0, n, [buf.data_ptr()] * 3, ws)
    G.gtr_ctx_check(ctx)
    assert np.array_equal(buf.cpu().numpy(), (o_out * np.uint64(3)).astype(np.uint64))


def test_branch_free_division_matches_ieee(G, ctx):
    """R-XS-div: wherever its guard accepts, the branch-free division of the
    warp-coherent loops returns exactly the IEEE quotient -- 2^28 pairs of raw
    bit patterns, lookup-shaped energy differences, neighbouring doubles and
    random exponents; the guard accepts the lookup-shaped pairs."""
    counts = torch.zeros(2, dtype=torch.uint64, device="cuda")
    n = 1 << 28
    G.gtr_ddiv_selftest(ctx, n, 20221002, counts)
    G.gtr_ctx_check(ctx)
    bad, acc = (int(x) for x in counts.cpu())
    assert bad == 0
    assert acc > n // 2          # all of the energy-shaped quarter and most of the rest


def test_sort_then_presorted(G, ctx, dev_small, small):
    """The two halves of the sorted mode: one sort, then the presorted
    lookups in several modes from the same workspace -- each identical to the
    oracle, per lookup."""
    t, P, o_out, o_v, n = small
    ws = torch.empty(G.gtr_xs_sorted_workspace_bytes(n), dtype=torch.uint8, device="cuda")
    G.gtr_xs_sort_lookups(ctx, dev_small.tables, 0, n, X.SEED_L, ws)
    for c in (G.cfg(G.SPMD, G.PL_STACK, 1, 256), G.cfg(G.CSM, G.PL_RUNTIME, 0, 128),
              G.cfg(G.GENERIC, G.PL_STACK, 1, 256), G.cfg(G.NATIVE, G.PL_STACK, 1, 256)):
        out = torch.zeros(18, dtype=torch.uint64, device="cuda")
        v, bufs = dev_small.verify_buffers(n)
        G.gtr_xs_lookup_presorted(ctx, c, dev_small.tables, 0, n, out, ws, v)
        G.gtr_ctx_check(ctx)
        _assert_same(out.cpu().numpy(), {k: b.cpu().numpy() for k, b in bufs.items()}, o_out, o_v)


def test_sorted_entry_points_reject_bad_workspace(G, ctx, dev_small):
    """Synchronous GTR_EINVAL (no launch) for a workspace that is too small or
    not 16-byte aligned, on every sorted-mode entry point."""
    n = 1000
    need = G.gtr_xs_sorted_workspace_bytes(n)
    small_ws = torch.empty(need - 16, dtype=torch.uint8, device="cuda")
    big = torch.empty(need + 64, dtype=torch.uint8, device="cuda")
    misaligned = big[8:8 + need]
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    h_out = torch.zeros(18, dtype=torch.uint64).pin_memory()
    c = G.cfg(G.SPMD, G.PL_STACK, 1, 256)
    for ws in (small_ws, misaligned):
        calls = [lambda: G.gtr_xs_sort_lookups(ctx, dev_small.tables, 0, n, X.SEED_L, ws),
                 lambda: G.gtr_xs_lookup_presorted(ctx, c, dev_small.tables, 0, n, out, ws),
                 lambda: G.gtr_xs_lookup_presorted_peers(ctx, c, dev_small.tables, 0, n, [out.data_ptr()], ws),
                 lambda: G.gtr_xs_lookup_sorted_host(ctx, c, dev_small.tables, G.gtr_xs_request(0, n, X.SEED_L),
                                                     h_out, ws),
                 lambda: G.gtr_xs_lookup_sorted(ctx, c, dev_small.tables, 0, n, X.SEED_L, out, ws)]
        for call in calls:
            with pytest.raises(G.GtrError):
                call()
    G.gtr_ctx_check(ctx)
    assert int(out.sum()) == 0


def test_sorted_mode_rejects_small_workspace(G, ctx, dev_small):
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    ws = torch.empty(1024, dtype=torch.uint8, device="cuda")
    with pytest.raises(G.GtrError):
        G.gtr_xs_lookup_sorted(ctx, G.cfg(), dev_small.tables, 0, 1000, X.SEED_L, out, ws)


# ---------------------------------------------------------------- fused combine (8(e), f1)
@pytest.mark.parametrize("mode", (0, 2, 3, 4))
def test_peer_combine_epilogue(G, ctx, dev_small, small, mode):
    """gtr_xs_lookup_peers adds every team's tallies into each listed buffer:
    listing the same buffer k times must give exactly k x the oracle (u64
    wrap-around), listing distinct buffers gives each the oracle's result."""
    t, P, o_out, o_v, n = small
    c = G.cfg(mode, G.PL_STACK, 1, 128)
    buf = torch.zeros(18, dtype=torch.uint64, device="cuda")
    G.gtr_xs_lookup_peers(ctx, c, dev_small.tables, 0, n, X.SEED_L, [buf.data_ptr()] * 3)
    G.gtr_ctx_check(ctx)
    assert np.array_equal(buf.cpu().numpy(), (o_out * np.uint64(3)).astype(np.uint64))
    bufs = torch.zeros((8, 18), dtype=torch.uint64, device="cuda")
    G.gtr_xs_lookup_peers(ctx, c, dev_small.tables, 0, n, X.SEED_L, [bufs[k].data_ptr() for k in range(8)])
    G.gtr_ctx_check(ctx)
    for k in range(8):
        assert np.array_equal(bufs[k].cpu().numpy(), o_out), k


def test_peer_combine_symmetric_memory_single_rank(G, ctx, dev_small, small):
    """The PeerCombine plumbing (torch symmetric memory, device barrier) at
    world size 1: three steps through the alternating slots."""
    import os
    import socket
    import torch.distributed as dist
    from paper_conf_cgo_hubercgtddcd22_b200.dist import PeerCombine
    t, P, o_out, o_v, n = small
    if not dist.is_initialized():
        s = socket.socket()
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
        s.close()
        os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK="0", WORLD_SIZE="1")
        dist.init_process_group("nccl", device_id=torch.device("cuda", 0))
    try:
        pc = PeerCombine(torch.device("cuda", 0))
        for _ in range(3):
            G.gtr_xs_lookup_peers(ctx, G.cfg(G.SPMD, G.PL_STACK, 1, 256), dev_small.tables, 0, n, X.SEED_L,
                                  pc.ptrs())
            res = pc.finish()
            assert np.array_equal(res.cpu().numpy(), o_out)
    finally:
        dist.destroy_process_group()


def test_variant_resources(G):
    info = G.gtr_query_variant(G.K_XS, G.cfg(G.SPMD, G.PL_STACK, 1, 256))
    assert info["block_threads"] == 256 and info["regs"] > 0 and info["num_teams"] > 0
    gen = G.gtr_query_variant(G.K_XS, G.cfg(G.GENERIC, G.PL_STACK, 1, 256))
    assert gen["block_threads"] == 288


@pytest.mark.slow
def test_large_config_bench_launch(G, ctx, orc):
    """Config 5 at full size (355 x 11,303, 17M lookups) in the launch
    configuration bench.py times: unionized grid exact, sampled index-grid rows
    exact, hash + tallies of all 17M lookups exact, 20,000 sampled lookups
    element-wise exact."""
    from paper_conf_cgo_hubercgtddcd22_b200.problems import XsDevice
    t = X.make_tables(355)
    P = orc.XsProblem(t)
    dev = XsDevice(ctx, t)
    assert np.array_equal(dev.egrid.cpu().numpy(), P.egrid)
    rows = np.random.default_rng(3).integers(0, P.n_union, 4000)
    rows = np.concatenate([rows, [0, 1, P.n_union - 2, P.n_union - 1]])
    assert np.array_equal(dev.index_grid[torch.from_numpy(rows).cuda()].cpu().numpy(), P.index_grid[rows])
    n = 17_000_000
    import os
    o_out, _ = P.run(0, n, X.SEED_L, os.cpu_count() or 8)
    for mode in (G.SPMD, G.NATIVE, G.CSM):
        out = torch.zeros(18, dtype=torch.uint64, device="cuda")
        G.gtr_xs_lookup(ctx, G.cfg(mode, G.PL_STACK, 1, 256), dev.tables, 0, n, X.SEED_L, out)
        G.gtr_ctx_check(ctx)
        assert np.array_equal(out.cpu().numpy(), o_out), mode
    # the sorted event mode (global counting sort + warp-coherent nuclide loops)
    ws = torch.empty(G.gtr_xs_sorted_workspace_bytes(n), dtype=torch.uint8, device="cuda")
    for mode in (G.SPMD, G.CSM):
        out = torch.zeros(18, dtype=torch.uint64, device="cuda")
        G.gtr_xs_lookup_sorted(ctx, G.cfg(mode, G.PL_STACK, 1, 256), dev.tables, 0, n, X.SEED_L, out, ws)
        G.gtr_ctx_check(ctx)
        assert np.array_equal(out.cpu().numpy(), o_out), ("sorted", mode)
    del ws
    first, m = 9_876_543, 20000
    o2, ov = P.run(first, m, X.SEED_L, 8, verify=True)
    out, v = _run(G, ctx, dev, G.cfg(G.SPMD, G.PL_STACK, 1, 256), first, m)
    _assert_same(out, v, o2, ov)


# ---------------------------------------------------------------- CUDA watermark of the bucketed schedule
@pytest.mark.parametrize("nt", (128, 256))
def test_native_bucketed_bit_exact(G, ctx, dev_small, small, nt):
    """GTR_F_NATIVE_BUCKETED: the bucketed/staged schedule as a plain CUDA
    kernel (no runtime) -- bit-identical lookups, also over a few teams with
    several chunks each and with ragged requests."""
    t, P, o_out, o_v, n = small
    c = G.cfg(G.NATIVE, G.PL_STACK, 1, nt, flags=G.F_NATIVE_BUCKETED)
    _assert_same(*_run(G, ctx, dev_small, c, 0, n), o_out, o_v)
    c2 = G.cfg(G.NATIVE, G.PL_STACK, 1, nt, num_teams=3, flags=G.F_NATIVE_BUCKETED)
    _assert_same(*_run(G, ctx, dev_small, c2, 0, n), o_out, o_v)
    for first, m in ((7, 1), (31337, 4097), (3, 12345)):
        _assert_same(*_run(G, ctx, dev_small, c2, first, m), *P.run(first, m, X.SEED_L, 4, verify=True))


def test_native_bucketed_sorted_and_grids(G, ctx, dev_small, dev_grid, small):
    t, P, o_out, o_v, n = small
    c = G.cfg(G.NATIVE, G.PL_STACK, 1, 256, flags=G.F_NATIVE_BUCKETED)
    out, v = _run_sorted(G, ctx, dev_small, c, 0, n)
    _assert_same(out, v, o_out, o_v)
    gt, dev = dev_grid
    out, v = _run(G, ctx, dev, c, 0, n)
    assert np.array_equal(out, o_out)
    assert np.array_equal(v["macro"].view(np.uint64), o_v["macro"].view(np.uint64))


def test_native_bucketed_rejects_plain_and_history(G, ctx, dev_small):
    out = torch.zeros(18, dtype=torch.uint64, device="cuda")
    for fl in (G.F_PLAIN, G.F_HISTORY):
        with pytest.raises(G.GtrError):
            G.gtr_xs_lookup(ctx, G.cfg(G.NATIVE, G.PL_STACK, 1, 256, flags=G.F_NATIVE_BUCKETED | fl),
                            dev_small.tables, 0, 1000, X.SEED_L, out)

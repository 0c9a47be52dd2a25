"""Pins for the XS oracle.

Each test checks oracle/xs.c against something other than itself: brute-force
stepping, exact rationals, python's bisect, numpy's sort/searchsorted,
scipy's linear interpolation, closed-form hashes of constructed tables.
"""
import bisect
from fractions import Fraction

import numpy as np
import pytest

import gtr_inputs.xs as X

A = 2806196910506780709
M = 1 << 63


def step(s):
    return (A * s + 1) % M


# ---------------------------------------------------------------- PIN-1
@pytest.mark.parametrize("seed", [0, 1, 1070, 42, M - 1, 123456789123456789])
def test_ff_equals_sequential_steps(orc, seed):
    s = seed % M
    want = {}
    checkpoints = set([0, 1, 2, 3, 5, 8, 64, 1000, 4097, 9999] + list(range(20)))
    for n in range(10001):
        if n in checkpoints:
            want[n] = s
        s = step(s)
    for n, v in want.items():
        assert orc.lcg_ff(seed, n) == v, n
        # next-state matches the definition too
        assert orc.lcg_next(v) == step(v)


def test_ff_composes(orc):
    rng = np.random.default_rng(5)
    for _ in range(200):
        a, b = (int(x) for x in rng.integers(0, 1 << 40, size=2))
        seed = int(rng.integers(0, 1 << 62))
        assert orc.lcg_ff(orc.lcg_ff(seed, a), b) == orc.lcg_ff(seed, a + b)


def test_uniform_is_exact_ratio(orc):
    s = 1070
    for _ in range(1000):
        d, s2 = orc.lcg_double(s)
        assert s2 == step(s)
        # u64 -> f64 rounds to nearest, / 2^63 is exact
        assert d == float(Fraction(s2, M))
        assert 0.0 <= d < 1.0
        s = s2


# ---------------------------------------------------------------- PIN-2
DIST = [Fraction(x) for x in ["0.140", "0.052", "0.275", "0.134", "0.154", "0.064",
                              "0.066", "0.055", "0.008", "0.015", "0.025", "0.013"]]


def seed_for_roll(r):
    """Seed whose next state is the 63-bit integer closest to r*2^63."""
    target = int(Fraction(r) * M) % M
    a_inv = pow(A, -1, M)
    return ((target - 1) * a_inv) % M


def test_pick_mat_cut_points(orc):
    # material i is chosen iff cum_{i-1} <= roll < cum_i with
    # cum_i = dist[1] + ... + dist[i]; dist[0] is never summed, so rolls
    # >= cum_11 = 0.861 give material 0 (the XSBench quirk kept verbatim).
    cum = [sum(DIST[1:i + 1], Fraction(0)) for i in range(12)]
    eps = Fraction(1, 10 ** 9)
    assert orc.pick_mat(seed_for_roll(Fraction(0)))[0] == 1
    for i in range(1, 12):
        assert orc.pick_mat(seed_for_roll(cum[i] - eps))[0] == i
        nxt = i + 1 if i < 11 else 0
        assert orc.pick_mat(seed_for_roll(cum[i] + eps))[0] == nxt
    assert orc.pick_mat(seed_for_roll(Fraction(999, 1000)))[0] == 0


def test_pick_mat_frequencies(orc):
    n = 200000
    counts = np.zeros(12)
    # sequential draws of the stream; chi-square against dist with p0 = .139
    s = 99
    for _ in range(n):
        m, s = orc.pick_mat(s)
        counts[m] += 1
    p = np.array([float(x) for x in DIST])
    p[0] = 1.0 - p[1:].sum()
    chi2 = (((counts - n * p) ** 2) / (n * p)).sum()
    assert chi2 < 40.0, (chi2, counts / n)


# ---------------------------------------------------------------- PIN-3
def test_grid_search_matches_bisect(orc):
    rng = np.random.default_rng(0)
    for trial in range(300):
        n = int(rng.integers(2, 40))
        a = np.sort(rng.integers(0, 12, size=n).astype(np.float64))   # duplicates
        for q in list(a) + [-1.0, 100.0, a[0], a[-1]] + list(rng.uniform(-1, 13, 8)):
            want = min(max(bisect.bisect_right(list(a), q) - 1, 0), n - 2)
            assert orc.grid_search(a, q) == want, (a, q)


# ---------------------------------------------------------------- PIN-4
def _tiny(n_iso, n_gp, seed):
    t = X.make_tables(n_iso, n_gp, seed_t=seed, seed_c=seed + 1)
    return t


@pytest.mark.parametrize("n_iso,n_gp,seed", [(3, 5, 1), (4, 7, 2), (7, 3, 3), (13, 40, 4)])
def test_union_and_index_grid_closed_form(orc, n_iso, n_gp, seed):
    t = _tiny(n_iso, n_gp, seed)
    P = orc.XsProblem(t)
    energies = t["grid"][:, :, 0]
    assert np.array_equal(P.egrid, np.sort(energies.ravel()))
    for u in range(P.n_union):
        for n in range(n_iso):
            cnt = np.searchsorted(energies[n], P.egrid[u], side="right")
            want = min(max(cnt - 1, 0), n_gp - 2)
            assert P.index_grid[u, n] == want


def test_index_grid_duplicates_hand_worked(orc):
    # nuclide 0 energies (0.1, 0.2, 0.2, 0.5), nuclide 1 (0.2, 0.3, 0.6, 0.7).
    # egrid = .1 .2 .2 .2 .3 .5 .6 .7.  The sequential rule advances at most
    # one step per union point, so nuclide 0 reaches index 1 at the first .2
    # and index 2 at the second .2 (worked by hand, tests/golden/xs_dup_index.txt).
    golden = np.loadtxt(__file__.replace("test_oracle_xs.py", "golden/xs_dup_index.txt"),
                        dtype=np.int32, comments="#")
    g = np.zeros((2, 4, 6))
    g[0, :, 0] = [0.1, 0.2, 0.2, 0.5]
    g[1, :, 0] = [0.2, 0.3, 0.6, 0.7]
    t = {"grid": g, "n_iso": 2, "n_gp": 4, "num_nucs": np.array([2] * 12, np.int32),
         "mats": np.tile(np.array([0, 1], np.int32), (12, 1)), "concs": np.ones((12, 2))}
    P = orc.XsProblem(t)
    assert np.array_equal(P.index_grid, golden)


# ---------------------------------------------------------------- PIN-5/6
def _energies_and_seeds(seed, n):
    """E_i and the post-energy state for lookups i < n by plain stepping."""
    out = []
    s = seed
    for i in range(n):
        s1 = step(s)
        out.append((float(Fraction(s1, M)), s1))
        s = step(step(s))
    return out


def test_lookup_against_library_interpolation(orc):
    from scipy.interpolate import interp1d
    t = X.make_tables(68, 1000)
    P = orc.XsProblem(t)
    n = 1500
    out, v = P.run(0, n, X.SEED_L, 1, verify=True)
    Es = _energies_and_seeds(X.SEED_L, n)
    g = t["grid"]
    interps = [interp1d(g[k, :, 0], g[k, :, 1:6].T, kind="linear", fill_value="extrapolate",
                        assume_sorted=True) for k in range(68)]
    eg = list(P.egrid)
    for i in range(n):
        E, s1 = Es[i]
        mat = int(v["mat"][i])
        assert mat == orc.pick_mat(s1)[0]
        assert int(v["u"][i]) == min(max(bisect.bisect_right(eg, E) - 1, 0), len(eg) - 2)
        want = np.zeros(5)
        for j in range(int(t["num_nucs"][mat])):
            nuc = int(t["mats"][mat, j])
            want += t["concs"][mat, j] * interps[nuc](E)
        np.testing.assert_allclose(v["macro"][i], want, rtol=1e-12, atol=1e-14)
        assert int(v["am"][i]) == int(np.argmax(v["macro"][i]))
    # hash / tally invariants
    assert out[0] == sum(int(a) + 1 for a in v["am"])
    assert out[1:13].sum() == n and out[13:18].sum() == n
    assert out[0] == sum((k + 1) * int(out[13 + k]) for k in range(5))


def test_interpolation_hits_gridpoint_exactly(orc):
    # E at or above a nuclide's last energy -> k = n_gp-2 (clamp), hi = last
    # point; if E == hi.e then f == 0 and every channel equals hi exactly.
    Es = _energies_and_seeds(X.SEED_L, 4)
    E0 = Es[0][0]
    t = X.make_tables(3, 50, seed_t=11)
    g = t["grid"]
    g[:, -1, 0] = E0                                 # last energy == E of lookup 0
    g[:, :-1, 0] = np.sort(g[:, :-1, 0] * E0 * 0.999, axis=1)
    t["num_nucs"][:] = 1
    t["mats"][:, 0] = [i % 3 for i in range(12)]
    t["concs"][:, 0] = 1.0
    P = orc.XsProblem(t)
    mat, u, macro, am = P.lookup(0, X.SEED_L)
    nuc = int(t["mats"][mat, 0])
    assert np.array_equal(macro, g[nuc, -1, 1:6])


# ---------------------------------------------------------------- PIN-7
@pytest.mark.parametrize("dominant,mult", [(0, 1), (4, 5), (2, 3)])
def test_hash_constructed_tables(orc, dominant, mult):
    t = X.constructed_tables(10, 400, dominant)
    P = orc.XsProblem(t)
    L = 3000
    out, v = P.run(0, L, X.SEED_L, 2, verify=True)
    assert out[0] == mult * L
    assert out[13 + dominant] == L


def test_nuclide_search_matches_bisect(orc):
    rng = np.random.default_rng(4)
    for _ in range(200):
        n = int(rng.integers(2, 60))
        g = np.zeros((n, 6))
        g[:, 0] = np.sort(rng.uniform(0, 1, n))
        lo = int(rng.integers(0, n - 1))
        hi = int(rng.integers(lo + 1, n))
        for q in list(rng.uniform(-0.1, 1.1, 6)) + [g[lo, 0], g[hi, 0]]:
            # lower-bound search inside [lo, hi]: last index in [lo, hi-1] with e <= q
            want = min(max(bisect.bisect_right(list(g[lo:hi + 1, 0]), q) - 1, 0), hi - lo - 1) + lo
            assert orc.nuclide_search(g, q, lo, hi) == want


def test_hash_index_closed_form(orc):
    t = X.make_tables(7, 300, seed_t=21)
    P = orc.XsProblem(t, grid_type=2, hash_bins=97)
    e = t["grid"][:, :, 0]
    for b in range(97):
        for n in range(7):
            cnt = np.searchsorted(e[n], b / 97.0, side="right")
            assert P.hash_index[b, n] == min(max(cnt - 1, 0), 300 - 2)


@pytest.mark.parametrize("n_iso,n_gp,bins", [(68, 2000, 10000), (13, 500, 37), (5, 50, 3)])
def test_grid_types_give_identical_lookups(orc, n_iso, n_gp, bins):
    # XSBench's three acceleration structures locate the same bracketing
    # interval (the last gridpoint <= E, clamped), so every lookup -- and the
    # hash -- must be identical to the unionized grid's (pinned above)
    t = X.make_tables(n_iso, n_gp, seed_t=n_gp)
    ref, vref = orc.XsProblem(t, grid_type=0).run(11, 3000, X.SEED_L, 2, verify=True)
    for gt in (1, 2):
        out, v = orc.XsProblem(t, grid_type=gt, hash_bins=bins).run(11, 3000, X.SEED_L, 2, verify=True)
        assert np.array_equal(out, ref)
        assert np.array_equal(v["macro"].view(np.uint64), vref["macro"].view(np.uint64))
        assert np.array_equal(v["mat"], vref["mat"]) and np.array_equal(v["am"], vref["am"])


def test_threads_do_not_change_results(orc):
    t = X.make_tables(68, 300)
    P = orc.XsProblem(t)
    a, va = P.run(5, 4000, X.SEED_L, 1, verify=True)
    b, vb = P.run(5, 4000, X.SEED_L, 7, verify=True)
    assert np.array_equal(a, b)
    for k in va:
        assert np.array_equal(va[k], vb[k])


def seed_with_first_draw(s1):
    """Lookup seed whose lookup-0 state after one LCG step is s1 (a * seed + 1 = s1)."""
    return (pow(A, -1, M) * ((s1 - 1) % M)) % M


@pytest.mark.parametrize("bins", [10000, 97, 1])
def test_energy_one_hash_bin_clamped(orc, bins):
    """E = 1.0 exactly (first draw 2^63 - 1 rounds up to 2^63, c1.1): the hash
    grid's bin E / du = hash_bins would be one row past the table (XSBench's
    own overread); the clamped last bin (DESIGN.md R-XS-hash1) must locate the
    same bracketing pair as the unionized grid -- the last pair of every
    nuclide, which a brute-force interpolation at E = 1.0 reproduces."""
    seed = seed_with_first_draw(M - 1)
    d, _ = orc.lcg_double(seed)
    assert d == 1.0
    t = X.make_tables(13, 200, seed_t=5)
    ref, vref = orc.XsProblem(t, grid_type=0).run(0, 64, seed, 1, verify=True)
    for gt in (1, 2):
        out, v = orc.XsProblem(t, grid_type=gt, hash_bins=bins).run(0, 64, seed, 1, verify=True)
        assert np.array_equal(out, ref)
        assert np.array_equal(v["macro"].view(np.uint64), vref["macro"].view(np.uint64))
    # brute force for lookup 0: every nuclide's last pair, hi - f (hi - lo), f = (hi.e - 1) / (hi.e - lo.e)
    mat = int(vref["mat"][0])
    g = t["grid"]
    want = np.zeros(5)
    for j in range(int(t["num_nucs"][mat])):
        nuc, c = int(t["mats"][mat, j]), float(t["concs"][mat, j])
        lo, hi = g[nuc, -2], g[nuc, -1]
        f = (hi[0] - 1.0) / (hi[0] - lo[0])
        want += (hi[1:6] - f * (hi[1:6] - lo[1:6])) * c
    assert np.allclose(vref["macro"][0], want, rtol=1e-13, atol=0)

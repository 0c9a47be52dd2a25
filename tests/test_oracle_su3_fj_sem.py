"""Pins for the SU3, fork/join and runtime-semantics oracles
(SURVEY.md 8(c) PIN-11, PIN-13)."""
import numpy as np
import pytest

import gtr_inputs.su3 as S


# ---------------------------------------------------------------- PIN-11
def test_su3_constant_closed_form(orc):
    A, B = S.make_lattice(3 ** 4, "constant")
    Cm = orc.su3_mat_nn(A, B)
    # 1/3 + 1/3 is exact, + 1/3 = 1 - 2^-54 rounds to even 1.0: every element 1.0
    assert np.all(Cm.real == 1.0) and np.all(Cm.imag == 0.0)
    assert np.all(Cm.real.reshape(-1, 36).sum(axis=1) == 36.0)


def test_su3_random_matches_library_and_group(orc):
    A, B = S.make_lattice(4 ** 4, "random")
    Cm = orc.su3_mat_nn(A, B, nthreads=3)
    want = np.einsum("sjkm,jml->sjkl", A, B)
    np.testing.assert_allclose(Cm, want, rtol=0, atol=2e-15)
    # SU(3) is a group: the product is unitary with det 1
    I3 = np.eye(3)
    CC = np.einsum("sjlk,sjlm->sjkm", Cm.conj(), Cm)
    assert np.abs(CC - I3).max() < 1e-13
    assert np.abs(np.linalg.det(Cm) - 1.0).max() < 1e-13


def test_su3_inputs_are_su3():
    A, B = S.make_lattice(2 ** 4, "random")
    M = A.reshape(-1, 3, 3)
    assert np.abs(np.einsum("nlk,nlm->nkm", M.conj(), M) - np.eye(3)).max() < 1e-13
    assert np.abs(np.linalg.det(M) - 1).max() < 1e-13


def test_su3_transposed_operand_detected(orc):
    # a plausible bug (B[j] transposed, or A*B vs B*A) changes the result
    A, B = S.make_lattice(2 ** 4, "random")
    Cm = orc.su3_mat_nn(A, B)
    assert np.abs(Cm - np.einsum("sjkm,jlm->sjkl", A, B)).max() > 1e-3
    assert np.abs(Cm - np.einsum("jkm,sjml->sjkl", B, A)).max() > 1e-3


# ---------------------------------------------------------------- PIN-13
@pytest.mark.parametrize("T,R", [(1, 1), (32, 7), (100, 50), (256, 1000)])
def test_fj_closed_forms(orc, T, R):
    for g in (0, 3):
        assert orc.fj_team(g, T, R, 0, 1) == R
        assert orc.fj_team(g, T, R, 1, 1) == (R * (R + 1) // 2) * (T * (T + 1) // 2)
        assert orc.fj_team(g, T, R, 2, 1) == T * (g * R * R + R * (R - 1) // 2)
    for K in (1, 4, 16):
        s = sum(((r % K) + 1) * (r + 1) for r in range(R))
        assert orc.fj_team(0, T, R, 1, K) == s * (T * (T + 1) // 2)


@pytest.mark.parametrize("body", [0, 1, 2])
def test_fj_host_team_equals_simulation(orc, body):
    T, R = 3, 500
    res, ns = orc.fj_host_team(T, R, body, 4)
    assert res == orc.fj_team(0, T, R, body, 4)
    assert ns > 0


def test_semantics_closed_forms(orc):
    G, T = 5, 64
    e = orc.sem_expected(0, G, T)
    for g in range(G):
        assert e[2 * g] == 2 * (1 + T)
        assert e[2 * g + 1] == (g + 1) + (g + G + 1) + 2 * (T * (T + 1) // 2)
    assert np.all(orc.sem_expected(1, G, T) == 42)
    assert list(orc.sem_expected(2, G, T)) == [3 * (g + 1) for g in range(G)]
    assert list(orc.sem_expected(3, G, T)) == [3 * (k + 1) for k in range(G * T)]
    e = orc.sem_expected(4, G, T)
    assert list(e[:G]) == [1] * G
    assert list(e[G:2 * G]) == [7 * g for g in range(G)]
    assert list(e[2 * G:]) == [7 * g + t for g in range(G) for t in range(T)]
    e = orc.sem_expected(5, G, T)
    assert list(e) == [1 + 20 + 100 + 10000 * T + 100000000 * t for g in range(G) for t in range(T)]
    # test 6 closed forms: omp_set_num_threads(T/2+1), then a region without
    # clause (n1 threads, nested serialized region inside), then num_threads(5)
    e = orc.sem_expected(6, G, T)
    n1 = T // 2 + 1
    A, B, Cc = e[:G * T].reshape(G, T), e[G * T:G * T + 5 * G].reshape(G, 5), e[G * T + 5 * G:].reshape(G, T)
    for g in range(G):
        for t in range(T):
            if t < n1:
                assert A[g, t] == t + 1000 * n1 + 10 ** 6 + 10 ** 7 + 10 ** 8 * n1
                assert Cc[g, t] == 20 + 100 + 1000 * t + 10 ** 7 * n1 + 10 ** 11 + 10 ** 12
            else:
                assert A[g, t] == 0 and Cc[g, t] == 0
        assert list(B[g]) == [t + 5000 + 10 ** 6 for t in range(5)]


@pytest.mark.parametrize("test", [7, 8])
@pytest.mark.parametrize("T", [32, 64, 128])
def test_semantics_schedules_closed_forms(orc, T, test):
    """test 7: static chunks dealt round robin (chunk k -> thread k mod n,
    OpenMP 5.1 sec. 2.11.4); dynamic and guided run each iteration once."""
    G = 3
    L, n = 3 * T + 7, (T // 2 + 1 if test == 7 else T // 2)
    e = orc.sem_expected(test, G, T)
    assert len(e) == 3 * G * L + G * T
    own, dyn, gui, chk = (e[:G * L].reshape(G, L), e[G * L:2 * G * L].reshape(G, L),
                          e[2 * G * L:3 * G * L].reshape(G, L), e[3 * G * L:].reshape(G, T))
    for g in range(G):
        for i in range(L):
            assert own[g, i] == (i // 3) % n + 1
        assert (dyn[g] == 1).all() and (gui[g] == 1).all()
        assert list(chk[g]) == [2 * L] * n + [0] * (T - n)

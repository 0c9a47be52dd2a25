"""GPU parity: SU3 mat_nn (config 3) vs the oracle -- bit-exact fp64 (both
sides round every product before the add, AMB-12), in every mode, placement
and fold, plus the constant-input closed form at full size."""
import itertools

import numpy as np
import pytest
import torch

import gtr_inputs.su3 as S
from gpu_common import G, ctx, pool, RUNTIME_MODES, PLACEMENTS  # noqa: F401

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def lattice(orc):
    A, B = S.make_lattice(6 ** 4 + 7, "random")     # ragged: not a multiple of any team size
    return A, B, orc.su3_mat_nn(A, B, nthreads=4)


def _run(G, ctx, cfg, A, B, iters=2):
    from paper_conf_cgo_hubercgtddcd22_b200.problems import su3_device
    dA, dB = su3_device(A, B)
    dC = torch.full_like(dA, float("nan"))
    G.gtr_su3_mat_nn(ctx, cfg, dA, dB, dC, A.shape[0], iters)
    G.gtr_ctx_check(ctx)
    return dC.cpu().numpy().view(np.complex128).reshape(A.shape)


@pytest.mark.parametrize("variant", list(itertools.product(RUNTIME_MODES, PLACEMENTS, (0, 1), (64, 128))),
                         ids=lambda v: "m%d-p%d-f%d-t%d" % v)
def test_su3_all_variants_bit_exact(G, ctx, lattice, variant):
    A, B, want = lattice
    m, p, f, nt = variant
    got = _run(G, ctx, G.cfg(m, p, f, nt, num_teams=97), A, B)
    assert np.array_equal(got.view(np.uint64), want.view(np.uint64))


@pytest.mark.parametrize("nt", (128, 256, 512))
def test_su3_native_bit_exact(G, ctx, lattice, nt):
    A, B, want = lattice
    got = _run(G, ctx, G.cfg(G.NATIVE, G.PL_STACK, 1, nt), A, B)
    assert np.array_equal(got.view(np.uint64), want.view(np.uint64))


def test_su3_full_lattice_constant_closed_form(G, ctx):
    sites = 32 ** 4
    A, B = S.make_lattice(sites, "constant")
    for mode in (G.SPMD, G.NATIVE):
        got = _run(G, ctx, G.cfg(mode, G.PL_STACK, 1, 128), A, B, iters=1)
        assert (got.real == 1.0).all() and (got.imag == 0.0).all()


@pytest.mark.parametrize("variant", list(itertools.product(RUNTIME_MODES, PLACEMENTS, (0, 1), (64, 128))),
                         ids=lambda v: "m%d-p%d-f%d-t%d" % v)
def test_su3_tma_all_variants_bit_exact(G, ctx, lattice, variant):
    """GTR_F_TMA: the sequential code streams 16-site tiles with bulk async
    copies (ragged last tile: 1303 sites = 81 x 16 + 7); same bits."""
    A, B, want = lattice
    m, p, f, nt = variant
    for teams in (0, 5):                     # one wave / few teams (many tiles per team)
        got = _run(G, ctx, G.cfg(m, p, f, nt, num_teams=teams, flags=G.F_TMA), A, B)
        assert np.array_equal(got.view(np.uint64), want.view(np.uint64)), teams


@pytest.mark.parametrize("nt", (128, 256, 512))
def test_su3_native_tma_bit_exact(G, ctx, lattice, nt):
    A, B, want = lattice
    for teams in (0, 3):
        got = _run(G, ctx, G.cfg(G.NATIVE, G.PL_STACK, 1, nt, num_teams=teams, flags=G.F_TMA), A, B)
        assert np.array_equal(got.view(np.uint64), want.view(np.uint64)), teams


def test_su3_tma_tiny_and_full(G, ctx, orc):
    for sites in (1, 15, 17):
        A, B = S.make_lattice(sites, "random")
        want = orc.su3_mat_nn(A, B)
        for mode in (G.SPMD, G.GENERIC, G.NATIVE):
            got = _run(G, ctx, G.cfg(mode, G.PL_STACK, 1, 128, flags=G.F_TMA), A, B)
            assert np.array_equal(got.view(np.uint64), want.view(np.uint64)), (sites, mode)
    A, B = S.make_lattice(32 ** 4, "constant")
    for mode in (G.SPMD, G.NATIVE):
        got = _run(G, ctx, G.cfg(mode, G.PL_STACK, 1, 128, flags=G.F_TMA), A, B, iters=1)
        assert (got.real == 1.0).all() and (got.imag == 0.0).all()

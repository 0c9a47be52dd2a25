"""GPU parity of the team runtime itself: fork/join (config 2) and the paper's
semantic programs (Figs. 1, 3, 5, 7, nested parallelism) in every mode,
placement and fold, against the oracle (exact integers)."""
import itertools

import numpy as np
import pytest
import torch

from gpu_common import G, ctx, pool, RUNTIME_MODES, PLACEMENTS  # noqa: F401

pytestmark = pytest.mark.gpu

FJ_VARIANTS = list(itertools.product(RUNTIME_MODES, PLACEMENTS, (0, 1), (32, 128, 256, 512)))


@pytest.mark.parametrize("variant", FJ_VARIANTS, ids=lambda v: "m%d-p%d-f%d-t%d" % v)
def test_forkjoin_all_variants(G, ctx, orc, variant):
    m, p, f, nt = variant
    teams, R = 37, 200
    for body, K in ((0, 1), (1, 1), (1, 16), (2, 1), (2, 5)):
        out = torch.zeros(teams, dtype=torch.uint64, device="cuda")
        G.gtr_forkjoin(ctx, G.cfg(m, p, f, nt, num_teams=teams), R, body, K, out)
        G.gtr_ctx_check(ctx)
        got = out.cpu().numpy()
        want = np.array([orc.fj_team(g, nt, R, body, K) for g in range(teams)], dtype=np.uint64)
        assert np.array_equal(got, want), (body, K)


@pytest.mark.parametrize("pl", PLACEMENTS)
@pytest.mark.parametrize("nt", (32, 256))
def test_forkjoin_one_barrier_broadcast(G, ctx, orc, pl, nt):
    teams, R = 20, 301
    out = torch.zeros(teams, dtype=torch.uint64, device="cuda")
    G.gtr_forkjoin(ctx, G.cfg(G.SPMD, pl, 1, nt, num_teams=teams, flags=G.F_BCAST_1BAR), R, 2, 3, out)
    G.gtr_ctx_check(ctx)
    want = np.array([orc.fj_team(g, nt, R, 2, 3) for g in range(teams)], dtype=np.uint64)
    assert np.array_equal(out.cpu().numpy(), want)


def test_barrier_floor_runs(G, ctx):
    out = torch.zeros(148, dtype=torch.uint64, device="cuda")
    G.gtr_barrier_floor(ctx, G.cfg(thread_limit=256, num_teams=148), 100, out)
    G.gtr_ctx_check(ctx)
    assert (out.cpu().numpy() > 0).all()


def test_generic_registers_exceed_csm_and_spmd(G):
    """P:593-597 (fn. 4): function pointers add spurious call edges that raise
    the register count; the custom state machine removes them."""
    r = {m: G.gtr_query_variant(G.K_FORKJOIN, G.cfg(m, G.PL_SHARED_STATIC, 1, 128))["regs"]
         for m in (G.GENERIC, G.GENERIC_CASCADE, G.CSM, G.SPMD)}
    assert r[G.GENERIC] > r[G.CSM] and r[G.GENERIC_CASCADE] > r[G.CSM], r
    assert r[G.SPMD] < r[G.GENERIC], r


SEM_VARIANTS = list(itertools.product(RUNTIME_MODES, PLACEMENTS, (0, 1), (64, 128)))


@pytest.mark.parametrize("variant", SEM_VARIANTS, ids=lambda v: "m%d-p%d-f%d-t%d" % v)
def test_semantics_all_variants(G, ctx, orc, variant):
    m, p, f, nt = variant
    G_teams = 6
    for test in range(9):
        if test >= 5 and f == 1:
            # folding assumes no nesting and no thread-count ICV changes
            with pytest.raises(G.GtrError, match="not instantiated"):
                G.gtr_semantics(ctx, G.cfg(m, p, f, nt, num_teams=G_teams), test,
                                torch.zeros(10 ** 5, dtype=torch.uint64, device="cuda"), 10 ** 5)
            continue
        want = orc.sem_expected(test, G_teams, nt)
        extra = len(want) if test in (2, 3) else 0
        out = torch.zeros(len(want) + extra, dtype=torch.uint64, device="cuda")
        G.gtr_semantics(ctx, G.cfg(m, p, f, nt, num_teams=G_teams), test, out, out.numel())
        G.gtr_ctx_check(ctx)
        got = out.cpu().numpy()
        if test == 1 and p == G.PL_COALESCED and m == G.SPMD:
            # LLVM-12 unsound shortcut: in SPMD mode LLVM 12 puts
            # every globalized local in thread-private memory without checking
            # whether its address escapes, so each thread dereferences thread
            # 0's address in its OWN local window and reads 42 + t -- the
            # miscompile the paper removes.  Every other
            # placement, heap-to-stack included, must give the oracle's 42:
            # heap-to-stack is illegal for the escaping Lcl.
            assert np.array_equal(got, want + np.tile(np.arange(nt, dtype=np.uint64), G_teams))
            continue
        assert np.array_equal(got[:len(want)], want), test
        if test in (2, 3):
            flags = got[len(want):]
            # LLVM 12 scheme: a converged warp in a parallel region (Fig. 5c)
            # gets a warp SoA on the shared-memory warp stack; the lone main
            # thread (Fig. 5b) and SPMD (private shortcut) do not
            in_shared = p in (G.PL_RUNTIME, G.PL_SHARED_STATIC, G.PL_STACK) or (
                p == G.PL_COALESCED and m != G.SPMD and test == 3)
            assert (flags == (1 if in_shared else 0)).all(), (test, flags[:4])


@pytest.mark.parametrize("pl", PLACEMENTS)
def test_fig7_separate_guards_same_result(G, ctx, orc, pl):
    want = orc.sem_expected(4, 6, 64)
    for flags in (0, G.F_SEPARATE_GUARDS):
        out = torch.zeros(len(want), dtype=torch.uint64, device="cuda")
        G.gtr_semantics(ctx, G.cfg(G.SPMD, pl, 1, 64, num_teams=6, flags=flags), 4, out, out.numel())
        G.gtr_ctx_check(ctx)
        assert np.array_equal(out.cpu().numpy(), want)


@pytest.mark.parametrize("kind", (0, 1), ids=("soft_barrier", "mbarrier"))
def test_watchdog_trips(G, ctx, kind):
    """A kernel whose wait can never complete (a software barrier one arrival
    short; an mbarrier phase nobody completes) finishes once the watchdog's
    spin limit is reached and reports the hang through the error word
    (GTR_EDEVICE) instead of hanging the GPU; the context is usable after."""
    G.gtr_ctx_set_spin_limit(ctx, 20000)
    try:
        G.gtr_watchdog_selftest(ctx, kind)
        with pytest.raises(G.GtrError, match="device-side"):
            G.gtr_ctx_check(ctx)
    finally:
        G.gtr_ctx_set_spin_limit(ctx, 0)
    G.gtr_ctx_check(ctx)                         # cleared
    out = torch.zeros(4, dtype=torch.uint64, device="cuda")
    G.gtr_forkjoin(ctx, G.cfg(G.SPMD, G.PL_STACK, 1, 128, num_teams=4), 10, 0, 1, out)
    G.gtr_ctx_check(ctx)
    assert (out.cpu().numpy() == 10).all()

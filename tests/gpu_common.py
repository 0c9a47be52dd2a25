"""Shared helpers of the -m gpu tests (all compute goes through libgtr.so)."""
import itertools

import pytest

RUNTIME_MODES = (0, 1, 2, 3)       # GENERIC, CASCADE, CSM, SPMD
PLACEMENTS = (0, 1, 2, 3, 4)       # RUNTIME, GLOBAL, SHARED_STATIC, STACK, COALESCED (LLVM 12)


def all_variants(nts):
    """(mode, placement, fold, thread_limit) for every runtime-mode variant."""
    return list(itertools.product(RUNTIME_MODES, PLACEMENTS, (0, 1), nts))


def vid(v):
    m, p, f, t = v
    return f"m{m}-p{p}-f{f}-t{t}"


@pytest.fixture(scope="session")
def G():
    import torch
    assert torch.cuda.is_available(), "gpu tests need a CUDA device"
    from paper_conf_cgo_hubercgtddcd22_b200 import gtr
    return gtr


@pytest.fixture(scope="session")
def pool():
    import torch
    # 256 MiB fallback pool for globalized variables (GTR_PL_GLOBAL and
    # shared-stack overflow)
    return torch.zeros(256 << 20, dtype=torch.uint8, device="cuda")


@pytest.fixture(scope="session")
def ctx(G, pool):
    c = G.gtr_ctx_create(0, pool.data_ptr(), pool.numel())
    yield c
    G.gtr_ctx_destroy(c)

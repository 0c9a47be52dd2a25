"""World-size-2 gloo tests of the N > 1 host path: weak-scaling
shards of the global lookup range, all-reduce of the 18 u64 results.  The
per-rank results come from the oracle (CPU); the combined hash must equal the
oracle's over the union of the ranges, for any world size."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import gtr_inputs.xs as X


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, ws, port, per_rank, q):
    import torch.distributed as dist
    import oracle
    from paper_conf_cgo_hubercgtddcd22_b200.dist import shard_range, combine_results, max_over_ranks
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    t = X.make_tables(12, 200, seed_t=5, seed_c=6)
    P = oracle.XsProblem(t)
    first, n = shard_range(rank, ws, per_rank)
    out_np, _ = P.run(first, n, X.SEED_L, 1)
    out = torch.from_numpy(out_np.copy())           # u64 [18]
    combine_results(out)
    tm = max_over_ranks(torch.tensor([float(rank + 1)], dtype=torch.float64))
    if rank == 0:
        q.put((out.numpy().copy(), float(tm[0])))
    dist.destroy_process_group()


@pytest.mark.parametrize("ws", [2, 3])
def test_sharded_hash_equals_union(orc, ws):
    per_rank = 1500
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, ws, port, per_rank, q)) for r in range(ws)]
    for p in procs:
        p.start()
    got, tmax = q.get(timeout=120)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    t = X.make_tables(12, 200, seed_t=5, seed_c=6)
    want, _ = orc.XsProblem(t).run(0, ws * per_rank, X.SEED_L, 1)
    assert np.array_equal(got, want)
    assert tmax == float(ws)


def test_shard_and_split_ranges():
    from paper_conf_cgo_hubercgtddcd22_b200.dist import shard_range, split_range
    assert shard_range(3, 8, 17_000_000) == (51_000_000, 17_000_000)
    parts = [split_range(10, 1001, r, 4) for r in range(4)]
    assert parts[0][0] == 10 and sum(n for _, n in parts) == 1001
    assert all(parts[i][0] + parts[i][1] == parts[i + 1][0] for i in range(3))
    with pytest.raises(ValueError):
        shard_range(2, 2, 5)


def test_u64_wraparound_through_int64_view():
    # hashes are u64; the int64 view used for the collective must round-trip
    a = torch.tensor([2 ** 63 + 5], dtype=torch.uint64)
    v = a.view(torch.int64)
    assert v.view(torch.uint64)[0] == a[0]


def _worker_apps(rank, ws, port, q):
    """RS lookups and SU3 sites sharded over ranks."""
    import torch.distributed as dist
    import oracle
    import gtr_inputs.rs as RS
    import gtr_inputs.su3 as S
    from paper_conf_cgo_hubercgtddcd22_b200.dist import shard_range, site_shard, combine_results, gather_shards
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    t = RS.make_tables(n_nuc=20, avg_poles=60, avg_windows=6)
    first, n = shard_range(rank, ws, 40)
    out_np, _, _ = oracle.RsProblem(t).run(first, n, X.SEED_L, 1)
    rs = torch.from_numpy(out_np.copy())
    combine_results(rs)
    f, m = site_shard(rank, ws, 7)
    A, B = S.make_lattice(m, "random", first_site=f)       # this rank's shard only
    Cl = torch.from_numpy(oracle.su3_mat_nn(A, B).view(np.float64).copy())
    Cg = gather_shards(Cl)
    if rank == 0:
        q.put((rs.numpy().copy(), Cg.numpy().copy()))
    dist.destroy_process_group()


@pytest.mark.parametrize("ws", [2, 3])
def test_sharded_rs_and_su3_equal_global(orc, ws):
    import gtr_inputs.rs as RS
    import gtr_inputs.su3 as S
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_apps, args=(r, ws, port, q)) for r in range(ws)]
    for p in procs:
        p.start()
    rs, Cg = q.get(timeout=180)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    t = RS.make_tables(n_nuc=20, avg_poles=60, avg_windows=6)
    want, _, _ = orc.RsProblem(t).run(0, 40 * ws, X.SEED_L, 1)
    assert np.array_equal(rs, want)
    A, B = S.make_lattice(7 * ws, "random")                 # the global lattice
    assert np.array_equal(Cg, orc.su3_mat_nn(A, B).view(np.float64))


def _worker_pc(rank, ws, port, want, q):
    import torch.distributed as dist
    from paper_conf_cgo_hubercgtddcd22_b200.dist import PeerCombine
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    pc, why = PeerCombine.create_all_or_none(torch.device("cpu"), want=want[rank])
    q.put((rank, pc is None, why))
    dist.destroy_process_group()


@pytest.mark.parametrize("want", [(True, True), (True, False), (False, False)])
def test_peer_combine_all_or_none(want):
    """The fused combine is chosen by all ranks or by none (a MIN all-reduce of
    the per-rank setup results): here peer-memory setup fails (CPU tensors) or
    is not requested on some rank, and every rank must fall back to NCCL
    together, with a reason, instead of deadlocking on mismatched paths."""
    ws = len(want)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_pc, args=(r, ws, port, want, q)) for r in range(ws)]
    for p in procs:
        p.start()
    res = sorted(q.get(timeout=120) for _ in range(ws))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert all(none for _, none, _ in res)
    assert all(why for _, _, why in res)

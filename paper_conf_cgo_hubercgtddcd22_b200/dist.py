"""Multi-GPU plumbing for the sharded lookups and lattices (SURVEY.md 8(e),
NEXT f1).

Lookups are independent and defined by their global id, so the N > 1 path is
a partition of the id range plus one all-reduce of the 18 u64 results (hash +
12 material tallies + 5 argmax tallies).  Integer sums: the combined result is
bit-identical for every world size.  torch.distributed supplies the process
group (NCCL over NVLink on the GPU box, gloo in the CPU tests).
"""
import torch


def shard_range(rank, world_size, per_rank):
    """Weak scaling: rank r owns global lookup ids [r*per_rank, (r+1)*per_rank)."""
    if not (0 <= rank < world_size):
        raise ValueError("rank out of range")
    return rank * per_rank, per_rank


def split_range(first, n, rank, world_size):
    """Strong scaling: split [first, first+n) into world_size contiguous parts."""
    lo = first + n * rank // world_size
    hi = first + n * (rank + 1) // world_size
    return lo, hi - lo


def combine_results(out, group=None):
    """All-reduce (SUM) an 18-entry u64 result tensor in place.  u64 is summed
    through an int64 view: two's-complement addition wraps identically."""
    import torch.distributed as dist
    if out.dtype == torch.uint64:
        view = out.view(torch.int64)
    elif out.dtype == torch.int64:
        view = out
    else:
        raise TypeError("results must be u64/i64")
    dist.all_reduce(view, op=dist.ReduceOp.SUM, group=group)
    return out


def max_over_ranks(values, group=None):
    """Element-wise max of a small float64 tensor over ranks (timings)."""
    import torch.distributed as dist
    dist.all_reduce(values, op=dist.ReduceOp.MAX, group=group)
    return values


def site_shard(rank, world_size, sites_per_rank):
    """SU3 weak scaling: rank r owns lattice sites [r*S, (r+1)*S) of A and C;
    B (4 links) is replicated.  Sites are independent: no collective on the
    data path."""
    return shard_range(rank, world_size, sites_per_rank)


def gather_shards(local, group=None):
    """Concatenate every rank's shard along dim 0 (validation only -- the
    shards stay resident on their GPUs in the benchmark)."""
    import torch.distributed as dist
    parts = [torch.empty_like(local) for _ in range(dist.get_world_size(group))]
    dist.all_gather(parts, local.contiguous(), group=group)
    return torch.cat(parts, 0)


class PeerCombine:
    """The 18-u64 all-reduce of the sharded XS step fused into the lookup
    kernel (gtr_xs_lookup_peers): every rank's teams add their tallies
    straight into every rank's result buffer over NVLink peer memory
    (system-scope atomics), then one device-side barrier.  The buffers are a
    torch symmetric-memory allocation (peer mappings of each rank's slot);
    two slots alternate so the next step's slot is zeroed before the barrier
    that precedes anyone's next kernel.  Integer sums: bit-identical to the
    NCCL all-reduce for any world size.

    Per step:  ptrs() -> launch gtr_xs_lookup_peers(..., ptrs) -> finish()
    (zero the other local slot, barrier on the current stream) -> the local
    slot holds the combined result."""

    # a device barrier that waits longer than this traps (the process fails
    # loudly) instead of hanging the job; one step takes ~17 ms
    BARRIER_TIMEOUT_MS = 60_000

    def __init__(self, device, group=None, timeout_ms=None):
        import torch.distributed as dist
        import torch.distributed._symmetric_memory as symm_mem
        g = group or dist.group.WORLD
        self.timeout_ms = self.BARRIER_TIMEOUT_MS if timeout_ms is None else int(timeout_ms)
        self.buf = symm_mem.empty(36, dtype=torch.int64, device=device).view(2, 18)
        self.handle = symm_mem.rendezvous(self.buf, g.group_name)
        self.nranks = int(self.handle.world_size)
        self.buf.zero_()
        self.handle.barrier(0, self.timeout_ms)
        self.step = 0

    @classmethod
    def create_all_or_none(cls, device, group=None, want=True):
        """Every rank tries to set the fused combine up; it is used only if it
        succeeded on ALL ranks (a MIN all-reduce of the success flags), so the
        ranks can never pick different combine paths.  Returns (PeerCombine or
        None, reason)."""
        import torch.distributed as dist
        pc, why = None, None
        if want:
            try:
                pc = cls(device, group)
            except Exception as e:  # noqa: BLE001 -- any setup failure selects the NCCL path on every rank
                why = f"{type(e).__name__}: {e}"[:160]
        flag = torch.tensor([1 if pc is not None else 0], dtype=torch.int64, device=device)
        dist.all_reduce(flag, op=dist.ReduceOp.MIN, group=group)
        if int(flag[0]) != 1:
            return None, why or ("not requested" if not want else "peer-memory setup failed on another rank")
        return pc, None

    def ptrs(self):
        off = (self.step % 2) * 18 * 8
        return [int(p) + off for p in self.handle.buffer_ptrs]

    def finish(self):
        b = self.step % 2
        self.buf[1 - b].zero_()
        self.handle.barrier(0, self.timeout_ms)
        self.step += 1
        return self.buf[b].view(torch.uint64)

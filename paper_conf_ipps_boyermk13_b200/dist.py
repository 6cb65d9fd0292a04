"""Multi-GPU plumbing: contiguous candidate shards and the cross-rank min-loc.

Candidates are independent, so the path shards with no data exchange; the
only collective is the final min-loc of one 48-byte grophecy_best_result per
rank: an all-gather over torch.distributed (NCCL on GPUs,
gloo in the CPU tests) followed by the library's combine (the
grophecy_best_combine kernel on GPUs, grophecy_best_combine_host on CPU).
NCCL has no MINLOC reduction; gathering P x 48 bytes and reducing locally is
exact, order-independent and latency-bound (one small collective per query).
"""
import torch
import torch.distributed as dist

RESULT_WORDS = 6   # 48 bytes as int64


def shard_range(n, rank, world):
    """Records [floor(rN/P), floor((r+1)N/P)) go to rank r; their global
    indices are index_base = floor(rN/P) + i, so ties resolve globally."""
    return (n * rank) // world, (n * (rank + 1)) // world


class MinLoc:
    """Device buffers for one query: ``local`` (this rank's result, written by
    grophecy_best_async), ``result`` (the global best after combine()).

    NCCL (default): the 48-byte results are all-gathered device to device on
    the compute stream, then the combine kernel runs on every rank.  With a
    gloo process group (CPU collectives; used to exercise the multi-rank path
    on a single GPU) the gather goes through host memory."""

    def __init__(self, world, device="cuda", backend=None):
        from . import grophecy as G
        self.G = G
        self.world = world
        self.backend = backend or (dist.get_backend() if world > 1 else "nccl")
        self.local = torch.empty(RESULT_WORDS, dtype=torch.int64, device=device)
        if world > 1:
            self.gathered = torch.empty(RESULT_WORDS * world, dtype=torch.int64, device=device)
            self.result = torch.empty(RESULT_WORDS, dtype=torch.int64, device=device)
            if self.backend != "nccl":
                self.h_local = torch.empty(RESULT_WORDS, dtype=torch.int64)
                self.h_gathered = torch.empty(RESULT_WORDS * world, dtype=torch.int64)
        else:
            self.result = self.local

    def combine(self):
        if self.world == 1:
            return self.result
        if self.backend == "nccl":
            dist.all_gather_into_tensor(self.gathered, self.local)
        else:
            self.h_local.copy_(self.local)
            dist.all_gather_into_tensor(self.h_gathered, self.h_local)
            self.gathered.copy_(self.h_gathered, non_blocking=True)
        self.G.best_combine(self.gathered, self.world, self.result)
        return self.result


def minloc_host(local_result, group=None):
    """CPU (gloo) version: all-gather BestResult structs, combine on the host
    with grophecy_best_combine_host.  Used by the multi-process CPU tests and
    any host-side orchestration."""
    from . import grophecy as G
    import ctypes
    raw = bytes(local_result)
    t = torch.frombuffer(bytearray(raw), dtype=torch.int64).clone()
    world = dist.get_world_size(group)
    out = [torch.empty_like(t) for _ in range(world)]
    dist.all_gather(out, t, group=group)
    res = [G.BestResult.from_buffer_copy(o.numpy().tobytes()) for o in out]
    return G.best_combine_host(res)

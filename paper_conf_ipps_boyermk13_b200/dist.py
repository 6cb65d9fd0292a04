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


def striped_chunks(n, rank, world, stripes, align=512):
    """Rank r's records as ``stripes`` chunks j = r + P k (k < stripes) of the
    P * stripes equal parts of [0, n), bounds rounded down to ``align`` (whole
    512-record tiles) except the end.  Global indices are unchanged (each
    chunk is projected with index_base = its start), so ties resolve
    globally and the union over ranks is [0, n) exactly once."""
    parts = world * stripes

    def bound(j):
        return n if j >= parts else (n * j // parts) // align * align

    out = []
    for k in range(stripes):
        j = rank + world * k
        a, b = bound(j), bound(j + 1)
        if b > a:
            out.append((a, b))
    return out or [(0, 0)]


def stripe_layout(n, rank, world, stripes, align=4096):
    """Rank r's share of [0, n) as ONE batch of back-to-back stripes plus a
    contiguous tail.  The first world * stripes * L records
    (L = n / (world * stripes) rounded down to ``align``, whole sweep tiles)
    are cut into stripes of L; rank r holds stripes j = r + world * k
    (k < stripes), stored contiguously, so its local record i has global index
    r * L + (i // L) * (world * L) + i % L: grophecy_batch's stripe map with
    index_base = r * L, stripe_len = L, stripe_stride = world * L (one launch
    per rank whatever ``stripes`` is; every rank gets a slice of every
    skeleton of a skeleton-major workload).  The rest [world * stripes * L, n)
    is split contiguously (shard_range).  Returns (L, main_count, (tail_lo,
    tail_hi)); L = 0 (everything in the tail) when n is too small."""
    L = (n // (world * stripes)) // align * align
    main_end = world * stripes * L
    t_lo, t_hi = shard_range(n - main_end, rank, world)
    return L, stripes * L, (main_end + t_lo, main_end + t_hi)


def stripe_global_index(i, rank, world, L):
    """Global index of batch-local record i of the main stripe batch."""
    return rank * L + (i // L) * (world * L) + i % L


class MinLoc:
    """Device buffers for one query: ``local`` (this rank's result, written by
    grophecy_best_async), ``result`` (the global best after combine()).

    NCCL (default): the 48-byte results are all-gathered device to device on
    the compute stream, then the combine kernel runs on every rank.  With a
    gloo process group (CPU collectives; used to exercise the multi-rank path
    on a single GPU) the gather goes through host memory."""

    def __init__(self, world, device="cuda", backend=None, space=None):
        from . import grophecy as G
        self.G = G
        self.world = world
        self.backend = backend or (dist.get_backend() if world > 1 else "nccl")
        self.local = torch.empty(RESULT_WORDS, dtype=torch.int64, device=device)
        # NCCL: the library's own communicator and grophecy_best_allreduce_result
        # (the product path); its unique id travels over the torch process group
        self.space, self.comm, self.host = space, None, None
        if world > 1 and self.backend == "nccl" and space is not None:
            uid = [G.nccl_unique_id() if dist.get_rank() == 0 else None]
            dist.broadcast_object_list(uid, src=0)
            self.comm = G.NcclComm(world, dist.get_rank(), uid[0], torch.cuda.current_device())
        if world > 1:
            self.gathered = torch.empty(RESULT_WORDS * world, dtype=torch.int64, device=device)
            self.result = torch.empty(RESULT_WORDS, dtype=torch.int64, device=device)
            if self.backend != "nccl":
                self.h_local = torch.empty(RESULT_WORDS, dtype=torch.int64)
                self.h_gathered = torch.empty(RESULT_WORDS * world, dtype=torch.int64)
        else:
            self.result = self.local

    def allreduce(self):
        """Global best on the host via grophecy_best_allreduce_result (NCCL
        all-gather + combine kernel + 48-byte D2H; synchronises)."""
        rc, r = self.space.allreduce_result(self.local, self.comm)
        return r

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


# ---------------------------------------------------------------------------
# Best transformation per group across shards ("cross-
# shard groups need a neighbour fix-up").  A group (maximal run of equal
# (skeleton, nx, ny, iters)) may straddle shard boundaries; the rank holding
# its first record reports it, merged over every continuation, and the later
# ranks drop their continuation pieces.  Only the boundary groups move: each
# rank contributes (n, first key, last key, first group, last group, n_groups).
def record_key(skx, nx, ny, iters):
    """Group key of one record (skeleton, nx, ny, iters)."""
    return (int(skx) >> 16, int(nx), int(ny), int(iters))


def shard_group_fixups(infos):
    """infos[r] = (n_records, first_key, last_key, first_group, last_group,
    n_groups) of rank r in shard order (groups as GroupResult; keys None for
    empty shards).  Returns per rank {"drop_first": bool, "last": GroupResult
    or None (replacement of the rank's last group)}.  Pure host logic; the
    merge itself is grophecy_group_merge_host."""
    from . import grophecy as G
    fix = [{"drop_first": False, "last": None} for _ in infos]
    open_r, open_key, acc = None, None, None
    for r, (n, fk, lk, fg, lg, ng) in enumerate(infos):
        if n == 0 or ng == 0:
            continue
        if open_r is not None and fk == open_key:
            acc = G.group_merge_host(acc, fg)
            fix[r]["drop_first"] = True
            fix[open_r]["last"] = acc
            if ng == 1:
                continue        # the whole shard continued the open group
        open_r, open_key, acc = r, lk, lg
    return fix


def apply_group_fixup(groups, fix):
    """Apply one rank's fix-up to its local list of GroupResult."""
    groups = list(groups)
    if fix["drop_first"]:
        groups = groups[1:]
    if fix["last"] is not None:
        groups[-1] = fix["last"]
    return groups


def fix_shard_groups(groups, n, first_key, last_key, group=None):
    """Collective (all ranks): exchange the boundary groups and return this
    rank's fixed list.  `groups` = this shard's GroupResult list."""
    from . import grophecy as G
    ng = len(groups)
    mine = (n, first_key, last_key, bytes(groups[0]) if ng else None,
            bytes(groups[-1]) if ng else None, ng)
    world = dist.get_world_size(group)
    allinfo = [None] * world
    dist.all_gather_object(allinfo, mine, group=group)
    infos = []
    for (nn, fk, lk, fg, lg, g) in allinfo:
        infos.append((nn, fk, lk, G.GroupResult.from_buffer_copy(fg) if fg else None,
                      G.GroupResult.from_buffer_copy(lg) if lg else None, g))
    fix = shard_group_fixups(infos)
    return apply_group_fixup(groups, fix[dist.get_rank(group)])


def group_best_sharded(space, pc, rec, index_base, group=None):
    """grophecy_group_best on this rank's shard (device records, global
    index_base) plus the cross-shard fix-up.  Returns this rank's groups."""
    rc, ng, groups = space.group_best(pc, rec, index_base=index_base)
    n = rec.n
    if n:
        ends = [[int(getattr(rec, f)[i].item()) & 0xffffffff for f in ("skx", "nx", "ny", "iters")]
                for i in (0, n - 1)]
        fk, lk = record_key(*ends[0]), record_key(*ends[1])
    else:
        fk = lk = None
    return fix_shard_groups(groups, n, fk, lk, group)

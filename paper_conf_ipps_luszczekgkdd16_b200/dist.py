"""Multi-GPU combine (§X-B: parallelise the
outermost loop nests).

One process per GPU (torchrun).  Every rank runs levels L1-L4 of the prefix
stage (replicated) and enumerates its own contiguous canonical shard -- a
work-balanced range of L4 survivors and everything below them -- through the
C ABI (beast_enumerate(rank, world)); the library never communicates.  This
module does the one exchange the method has:

  all_gather of the per-rank survivor counts -> exclusive scan = each shard's
  global offset; all_reduce(sum) of the statistics; gather of the survivor
  records to rank 0 in rank order (= canonical order), with point-to-point
  transfers into rank 0's buffer at the scanned offsets (NCCL over NVLink on
  GPUs, gloo in the CPU tests).

The functions take and return torch tensors on whatever device the process
group uses; they contain no enumeration logic.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

STAT_LEN = 15 + 12 + 4 + 4   # visits, rejected, survivors, prefixes, valid_a, tuples, formed[2], checked[2]


class ReplicaMismatch(RuntimeError):
    """The ranks' redundantly computed L1-L4 lists differ."""


def _dev():
    return torch.device("cuda", torch.cuda.current_device()) \
        if dist.is_initialized() and dist.get_backend() == "nccl" else torch.device("cpu")


def stats_to_tensor(st: dict, device=None) -> torch.Tensor:
    v = list(st["visits"]) + list(st["rejected"]) + [st["survivors"], st["prefixes"], st["valid_a"], st["tuples"]]
    v += list(st.get("formed", (0, 0))) + list(st.get("checked", (0, 0)))
    return torch.tensor(v, dtype=torch.int64, device=device or _dev())


def tensor_to_stats(t: torch.Tensor) -> dict:
    v = [int(x) for x in t.cpu().tolist()]
    st = dict(visits=v[:15], rejected=v[15:27], survivors=v[27], prefixes=v[28], valid_a=v[29], tuples=v[30],
              formed=v[31:33], checked=v[33:35])
    st["points"] = sum(st["visits"])
    return st


def _u64_to_i64(x: int) -> int:
    return x - (1 << 64) if x >= (1 << 63) else x


def check_replicas(l4_digest: int, world: int, device=None) -> list:
    """every rank computes levels L1-L4 redundantly; all-gather
    the 64-bit digest of each rank's L4 survivor list (beast_stats.l4_digest
    / Space.last_l4_digest) and raise ReplicaMismatch unless all ranks
    agree.  Returns the gathered digests (unsigned)."""
    if world <= 1 or not dist.is_initialized():
        return [int(l4_digest)]
    dev = device or _dev()
    mine = torch.tensor([_u64_to_i64(int(l4_digest))], dtype=torch.int64, device=dev)
    allv = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in range(world)]
    dist.all_gather(allv, mine)
    got = [int(x.item()) & ((1 << 64) - 1) for x in allv]
    if len(set(got)) != 1:
        raise ReplicaMismatch("L4 survivor lists differ across ranks: digests %s" % ["0x%016x" % d for d in got])
    return got


def combine_stats(st: dict, world: int) -> dict:
    """Sum the per-shard statistics over all ranks (each level L1..L6 is
    charged to rank 0 only by the library, so the sum is the whole space);
    the L4 digest is checked equal across ranks (check_replicas) instead of
    summed."""
    if world <= 1 or not dist.is_initialized():
        out = dict(st)
        out["points"] = sum(st["visits"])
        return out
    if "l4_digest" in st:
        check_replicas(st["l4_digest"], world)
    t = stats_to_tensor(st)
    dist.all_reduce(t, op=dist.ReduceOp.SUM)
    out = tensor_to_stats(t)
    if "l4_digest" in st:
        out["l4_digest"] = st["l4_digest"]
    return out


def shard_offsets(n_local: int, world: int, device=None) -> list:
    """all_gather of the shard sizes; returns [offset_0, ..., offset_world]
    (exclusive scan, offset_world = total)."""
    if world <= 1 or not dist.is_initialized():
        return [0, n_local]
    dev = device or _dev()
    mine = torch.tensor([n_local], dtype=torch.int64, device=dev)
    allc = [torch.zeros(1, dtype=torch.int64, device=dev) for _ in range(world)]
    dist.all_gather(allc, mine)
    counts = [int(c.item()) for c in allc]
    offs = [0]
    for c in counts:
        offs.append(offs[-1] + c)
    return offs


def gather_records(local: torch.Tensor, gathered, world: int, root: int = 0) -> int:
    """Gather every rank's (n_r, 2) record shard into `gathered` on `root` at
    its canonical offset.  Returns the global count (on every rank)."""
    n = int(local.shape[0])
    offs = shard_offsets(n, world, local.device)
    total = offs[-1]
    if world <= 1 or not dist.is_initialized():
        if gathered is not None and gathered.data_ptr() != local.data_ptr() and n:
            gathered[:n].copy_(local)
        return total
    rank = dist.get_rank()
    lv = local.view(torch.int64) if local.dtype == torch.uint64 else local
    ops = []
    if rank == root:
        gv = gathered.view(torch.int64) if gathered.dtype == torch.uint64 else gathered
        for r in range(world):
            a, b = offs[r], offs[r + 1]
            if b == a:
                continue
            if r == root:
                gv[a:b].copy_(lv)
            else:
                ops.append(dist.P2POp(dist.irecv, gv[a:b], r))
    elif n:
        ops.append(dist.P2POp(dist.isend, lv.contiguous(), root))
    if ops:
        for req in dist.batch_isend_irecv(ops):
            req.wait()
    return total


def enumerate_distributed(space, gather=False, stats=False, stream=None) -> dict:
    """Enumerate this rank's shard with the library and combine.  Every rank
    must pass the same `gather`.  Returns dict(local=records of this shard,
    offset=its global offset, total=global count, gathered=the full canonical
    list on rank 0 when gather=True, stats=summed stats when stats=True)."""
    world = dist.get_world_size() if dist.is_initialized() else 1
    rank = dist.get_rank() if dist.is_initialized() else 0
    if stats:
        rec, st = space.enumerate(rank=rank, world=world, stream=stream, stats=True)
    else:
        rec, st = space.enumerate(rank=rank, world=world, stream=stream), None
    offs = shard_offsets(int(rec.shape[0]), world, rec.device)
    out = dict(local=rec, offset=offs[rank], total=offs[-1], gathered=None)
    if gather:
        buf = torch.empty((max(offs[-1], 1), 2), dtype=rec.dtype, device=rec.device) if rank == 0 else None
        gather_records(rec, buf, world)
        out["gathered"] = buf[:offs[-1]] if buf is not None else None
    if stats:
        out["stats"] = combine_stats(st, world)
    return out


class FusedGather:
    """fused survivor gather.

    Instead of enumerating into a local buffer and then gathering with NCCL,
    every rank stages its shard (beast_enumerate_stage: the pass up to the
    canonical tuple list, its record count into a device word), the counts
    are all-gathered (NCCL, 8 bytes per rank), and every rank's write-out
    kernel stores its records directly into rank 0's buffer at the shard's
    global offset (beast_write_at), the buffer being symmetric memory mapped
    into every rank over NVLink.  A symmetric-memory barrier then makes the
    list complete on rank 0.  With one process (no process group) the buffer
    is an ordinary local tensor.  `capacity` = records the list may hold
    (the whole space's survivors)."""

    def __init__(self, capacity: int, device=None, group=None):
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.device = device or torch.device("cuda", torch.cuda.current_device())
        self.capacity = max(int(capacity), 1)
        self.group = group
        self.hdl = None
        if self.world > 1:
            import torch.distributed._symmetric_memory as symm_mem
            self.buf = symm_mem.empty((self.capacity, 2), dtype=torch.int64, device=self.device)
            self.hdl = symm_mem.rendezvous(self.buf, group if group is not None else dist.group.WORLD)
            self.root_ptr = int(self.hdl.buffer_ptrs[0])   # rank 0's buffer, mapped into this process
        else:
            self.buf = torch.empty((self.capacity, 2), dtype=torch.int64, device=self.device)
            self.root_ptr = self.buf.data_ptr()
        self.d_count = torch.zeros(1, dtype=torch.int64, device=self.device)
        self.d_counts = torch.zeros(self.world, dtype=torch.int64, device=self.device)

    def run(self, space, stream=None) -> int:
        """One fused enumeration + gather; returns the global record count.
        On rank 0, self.buf[:total] then holds the canonical list (int64 view
        of the (lo, hi) records).

        Order: stage (local) -> all-gather of the counts -> every rank checks
        the total against the capacity (the same counts everywhere, so all
        ranks raise together and none is left waiting in a barrier) ->
        barrier (rank 0 has finished with the previous list before any rank
        overwrites it) -> write into rank 0's buffer -> barrier (the list is
        complete)."""
        from . import beast_enumerate_stage, beast_write_at
        beast_enumerate_stage(space.handle, self.d_count, self.rank, self.world, stream)
        if self.world > 1:
            dist.all_gather_into_tensor(self.d_counts, self.d_count, group=self.group)
        else:
            self.d_counts.copy_(self.d_count)
        total = int(self.d_counts.sum().item())
        if total > self.capacity:
            raise ValueError("fused gather: %d records exceed the buffer's capacity %d" % (total, self.capacity))
        if self.hdl is not None:
            self.hdl.barrier()
        beast_write_at(space.handle, self.root_ptr, self.capacity, self.d_counts, self.rank, self.world, stream)
        if self.hdl is not None:
            self.hdl.barrier()
        return total

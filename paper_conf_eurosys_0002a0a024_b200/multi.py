"""Multi-GPU plumbing for batches of independent vertex queries.

Vertex queries are independent: the source list is split into contiguous shards,
one per rank (each GPU holds a full replica of G and its Core Graphs), and the only exchange
is gathering the value rows to rank 0.  torch.distributed provides the transport (NCCL over
NVLink / NVSwitch on GPUs, gloo in the CPU tests); nothing here computes.
"""
from __future__ import annotations

import torch
import torch.distributed as dist


def shard(n_total: int, rank: int, world: int) -> tuple[int, int]:
    """[start, stop) of rank's contiguous shard; shard sizes differ by at most one."""
    if world <= 0 or not 0 <= rank < world:
        raise ValueError("bad rank / world size")
    base, extra = divmod(n_total, world)
    start = rank * base + min(rank, extra)
    return start, start + base + (1 if rank < extra else 0)


def gather_rows(values: torch.Tensor, rank: int, world: int, root_buffers=None, async_op: bool = False):
    """Gather every rank's [rows, n] value block to rank 0 (equal row counts per rank).

    root_buffers: on rank 0, a list of `world` tensors shaped like `values` (allocated here if
    None).  Returns (buffers on rank 0 / None elsewhere, work handle or None)."""
    if world == 1:
        return [values], None
    if rank == 0 and root_buffers is None:
        root_buffers = [torch.empty_like(values) for _ in range(world)]
    work = dist.gather(values, root_buffers if rank == 0 else None, dst=0, async_op=async_op)
    return (root_buffers if rank == 0 else None), work


def max_over_ranks(x: float, device=None) -> float:
    """Max of a host scalar over all ranks (timing is reported as the slowest rank)."""
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size() == 1:
        return x
    t = torch.tensor([x], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return float(t.item())


def hub_shard(K: int, rank: int, world: int) -> tuple[int, int]:
    """[begin, end) of the hubs whose Identify queries rank runs in a sharded CG build (NEXT-4)."""
    return shard(K, rank, world)


def merge_flags(flags: torch.Tensor, group=None) -> torch.Tensor:
    """OR of the ranks' Algorithm 1 edge flags (uint8 0/1): an all-reduce with MAX, in place
    (ncclAllReduce(ncclUint8, ncclMax) over NVLink on GPUs; gloo in the CPU tests)."""
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(flags, op=dist.ReduceOp.MAX, group=group)
    return flags


def build_sharded(graph, kind, K: int = 20, rank: int = 0, world: int = 1, group=None, **kw) -> dict:
    """Sharded Core Graph build (NEXT-4): every rank runs the Identify queries of
    its hub shard (cg_build_partial), the flags are OR-reduced across ranks, and every rank
    installs the same merged CG (cg_build_from_flags).  Algorithm 1 kinds only."""
    b, e = hub_shard(K, rank, world)
    flags = graph.build_partial(kind, K=K, hub_range=(b, e), **kw)
    merge_flags(flags, group)
    return graph.build_from_flags(kind, flags, K=K, **kw)


class GatherRing:
    """Double-buffered result gather to rank 0 (the path's single exchange step).

    Step i writes its value rows into slot i % slots and starts an asynchronous gather of them;
    before step i + slots rewrites that slot, ``acquire`` waits for step i's gather (a stream
    wait, no host sync), so a gather never reads a block that a later step is overwriting.
    Rank 0 gathers each slot into that slot's own root buffers.  Blocks travel as bytes, so any
    dtype works (uint16 / bit-packed narrow rows, uint32 rows)."""

    def __init__(self, rank: int, world: int, slots: int = 2):
        self.rank, self.world, self.slots = rank, world, slots
        self.works = [[] for _ in range(slots)]
        self.roots = [{} for _ in range(slots)]

    def acquire(self, slot: int) -> None:
        for w in self.works[slot]:
            w.wait()
        self.works[slot] = []

    def submit(self, slot: int, key, block: torch.Tensor) -> None:
        if self.world == 1:
            return
        raw = block.view(torch.uint8) if block.dtype != torch.uint8 else block
        bufs = None
        if self.rank == 0:
            bufs = self.roots[slot].get(key)
            if bufs is None or bufs[0].shape != raw.shape:
                bufs = [torch.empty_like(raw) for _ in range(self.world)]
                self.roots[slot][key] = bufs
        _, work = gather_rows(raw, self.rank, self.world, bufs, async_op=True)
        self.works[slot].append(work)

    def gathered(self, slot: int, key):
        """Rank 0: the world's blocks of `key` in `slot` (valid after acquire / drain)."""
        return self.roots[slot].get(key)

    def drain(self) -> None:
        for s in range(self.slots):
            self.acquire(s)

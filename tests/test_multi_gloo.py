"""World-size-2 gloo test of the multi-GPU host logic (sharding + gather to rank 0).

Each rank evaluates its shard of the sources (with the CPU oracle standing in for a GPU — the
CUDA path is exercised by the -m gpu tests) and the values are gathered to rank 0 with the same
`paper_conf_eurosys_0002a0a024_b200.multi` functions bench.py uses; rank 0 must hold exactly
the single-process result."""
import os
import socket
import sys

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, out_path):
    sys.path.insert(0, ROOT)
    import gen
    import oracle
    from paper_conf_eurosys_0002a0a024_b200 import multi

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n = 1 << 10
    src, dst, w = gen.rmat(n, 8 * n, seed=3)
    g = oracle.canonical_csr(n, src, dst, w)
    sources = gen.sample_sources(n, src, dst, 2 * world, seed=5)
    a, b = multi.shard(len(sources), rank, world)
    mine = torch.from_numpy(oracle.query_batch("sssp", g, sources[a:b]).view(np.int32))
    bufs, work = multi.gather_rows(mine, rank, world, async_op=True)
    work.wait()
    t = multi.max_over_ranks(float(rank))
    if rank == 0:
        full = torch.cat(bufs).numpy().view(np.uint32)
        np.save(out_path, full)
        assert t == world - 1
    dist.barrier()
    dist.destroy_process_group()


def test_shard_sizes():
    from paper_conf_eurosys_0002a0a024_b200 import multi
    for n in (0, 1, 7, 64, 129):
        for world in (1, 2, 3, 8):
            parts = [multi.shard(n, r, world) for r in range(world)]
            assert parts[0][0] == 0 and parts[-1][1] == n
            assert all(parts[i][1] == parts[i + 1][0] for i in range(world - 1))
            sizes = [b - a for a, b in parts]
            assert max(sizes) - min(sizes) <= 1
    with pytest.raises(ValueError):
        multi.shard(4, 2, 2)


def test_gather_world2(tmp_path):
    import gen
    import oracle
    out = str(tmp_path / "full.npy")
    mp.spawn(_worker, args=(2, _free_port(), out), nprocs=2, join=True)
    full = np.load(out)
    n = 1 << 10
    src, dst, w = gen.rmat(n, 8 * n, seed=3)
    g = oracle.canonical_csr(n, src, dst, w)
    sources = gen.sample_sources(n, src, dst, 4, seed=5)
    assert np.array_equal(full, oracle.query_batch("sssp", g, sources))


def _merge_worker(rank, world, port, out_path):
    sys.path.insert(0, ROOT)
    import gen
    import oracle
    from paper_conf_eurosys_0002a0a024_b200 import multi

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n, K = 1 << 10, 12
    src, dst, w = gen.rmat(n, 8 * n, w_max=31, seed=7)
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    hubs = oracle.hubs_topdeg(g, gr, K)
    b, e = multi.hub_shard(K, rank, world)
    # this rank's Identify queries (the CPU oracle stands in for cg_build_partial on a GPU)
    mine = torch.from_numpy(oracle.cg_alg1("sswp", g, gr, hubs[b:e], connectivity=False))
    multi.merge_flags(mine)
    if rank == 0:
        np.save(out_path, mine.numpy())
    dist.barrier()
    dist.destroy_process_group()


def test_sharded_core_graph_merge_world2(tmp_path):
    """NEXT-4: Algorithm 1 is a union over hubs, so marking half the hubs per rank and OR-ing
    the flags (all-reduce MAX over uint8) reproduces the single-process flags exactly."""
    import gen
    import oracle
    out = str(tmp_path / "flags.npy")
    mp.spawn(_merge_worker, args=(2, _free_port(), out), nprocs=2, join=True)
    n, K = 1 << 10, 12
    src, dst, w = gen.rmat(n, 8 * n, w_max=31, seed=7)
    g = oracle.canonical_csr(n, src, dst, w)
    gr = oracle.transpose(g)
    exp = oracle.cg_alg1("sswp", g, gr, oracle.hubs_topdeg(g, gr, K), connectivity=False)
    assert np.array_equal(np.load(out), exp)


def _ring_worker(rank, world, port, out_path):
    sys.path.insert(0, ROOT)
    from paper_conf_eurosys_0002a0a024_b200 import multi

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ring = multi.GatherRing(rank, world, slots=2)
    blocks = [torch.zeros((3, 5), dtype=torch.int16) for _ in range(2)]  # the two output slots
    seen = []
    for i in range(7):
        slot = i % 2
        ring.acquire(slot)  # step i-2's gather of this slot has finished
        if rank == 0 and i >= 2:  # ... so the root buffers hold step i-2's rows, whole
            seen.append([int(b.view(torch.int16)[0, 0]) for b in ring.gathered(slot, "k")])
        blocks[slot].fill_(100 * i + rank)  # step i overwrites its slot
        ring.submit(slot, "k", blocks[slot])
    ring.drain()
    if rank == 0:
        for i in (5, 6):
            seen.append([int(b.view(torch.int16)[0, 0]) for b in ring.gathered(i % 2, "k")])
        np.save(out_path, np.array(seen))
    dist.barrier()
    dist.destroy_process_group()


def test_gather_ring_slot_reuse_world2(tmp_path):
    """The bench's double-buffered gather (multi.GatherRing): a slot is rewritten only after the
    gather that read it finished, and rank 0's per-slot root buffers hold exactly the step that
    was gathered into them (no write-after-read race between step i's gather and step i+2)."""
    out = str(tmp_path / "seen.npy")
    mp.spawn(_ring_worker, args=(2, _free_port(), out), nprocs=2, join=True)
    seen = np.load(out)
    exp = np.array([[100 * i, 100 * i + 1] for i in range(7)])
    assert np.array_equal(seen, exp)

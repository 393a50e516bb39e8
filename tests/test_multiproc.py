"""World-size-2 (and 3) gloo tests of the multi-GPU host logic on CPU: seed sharding with
global ids + one reduce(SUM) of the int32-viewed maps reproduce the single-process map
bit for bit.  The per-rank tracker here is the oracle (test infrastructure); on GPUs the
same shard/reduce code drives libpt.so over NCCL (bench.py)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, block):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import phantom
        from paper_conf_ipps_xuzwrwxgxy12_b200 import sharding
        w = phantom.crossing(sigma=0.15, f_jitter=0.03, nseeds=48, particles_per_seed=60, nsamples=20)
        seeds, ids = sharding.shard_seeds(w.seeds, w.seed_ids, rank, world, block=block)
        assert seeds.shape[0] > 0  # every rank has work (block < 48 seeds / world)
        r = oracle.track(w.replace(seeds=seeds, seed_ids=ids))
        m = torch.from_numpy(r["map"].astype(np.uint32).view(np.int32).copy())
        sharding.reduce_map(m, dst=0)
        # uint32 wrap-around survives the int32 reduce: each rank adds 2^31 + rank to cell 0
        wrap = torch.tensor([np.int32(-2**31 + rank)], dtype=torch.int32)
        sharding.reduce_map(wrap, all_ranks=True)
        steps = torch.tensor([int(r["nsteps"].sum())], dtype=torch.int64)
        dist.all_reduce(steps)
        if rank == 0:
            full = oracle.track(w)
            q.put((m.numpy().view(np.uint32).copy(), full["map"].astype(np.uint32),
                   int(wrap[0].item()) & 0xFFFFFFFF, int(steps[0]), int(full["nsteps"].sum())))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,block", [(2, 0), (3, 0), (2, 5), (3, 4)])
def test_sharded_reduce_matches_single_process(world, block):
    """block 0: seed i -> rank i mod world; block > 0: Z-order blocks (the bench default,
    with a block small enough that every rank gets several blocks of the 48 seeds)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, block)) for r in range(world)]
    for p in procs:
        p.start()
    got, full, wrap, steps, full_steps = q.get(timeout=600)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert np.array_equal(got, full)
    assert steps == full_steps == int(full.sum(dtype=np.uint64))
    expect = sum((2**31 + r) for r in range(world)) & 0xFFFFFFFF
    assert wrap == expect


def test_shard_indices_partition():
    from paper_conf_ipps_xuzwrwxgxy12_b200 import sharding
    for n in (0, 1, 7, 100):
        for world in (1, 2, 3, 8):
            parts = [sharding.shard_indices(n, r, world) for r in range(world)]
            allp = np.sort(np.concatenate(parts)) if n else np.array([], np.int64)
            assert np.array_equal(allp, np.arange(n))
    with pytest.raises(ValueError):
        sharding.shard_indices(5, 2, 2)


def test_shard_blocks_partition_and_locality():
    """Block-interleaved Z-order sharding: the shards partition the seeds (every seed on
    exactly one rank, none twice), blocks are contiguous in Z-order, and the shard sizes
    differ by at most one block."""
    from paper_conf_ipps_xuzwrwxgxy12_b200 import sharding
    rng = np.random.default_rng(3)
    for n, world, block in ((0, 2, 4), (1, 3, 4), (1000, 1, 256), (1000, 3, 16), (5000, 8, 64), (777, 8, 256)):
        seeds = (rng.integers(0, 64, size=(n, 3)) + 0.5).astype(np.float32)
        parts = [sharding.shard_blocks(seeds, r, world, block) for r in range(world)]
        allp = np.sort(np.concatenate(parts)) if n else np.array([], np.int64)
        assert np.array_equal(allp, np.arange(n))
        sizes = [p.size for p in parts]
        assert max(sizes) - min(sizes) <= block
        perm = sharding.morton_order(seeds)
        pos = np.empty(n, np.int64)
        pos[perm] = np.arange(n)
        for r, p in enumerate(parts):  # rank r holds exactly the Z-order blocks b = r mod world
            assert np.all((pos[p] // block) % world == r)
    # the Z-order agrees with the spec: (x, y, z) bits interleaved x lowest
    s = np.array([[1.5, 0.5, 0.5], [0.5, 1.5, 0.5], [0.5, 0.5, 1.5], [0.5, 0.5, 0.5]], np.float32)
    assert list(sharding.morton_order(s)) == [3, 0, 1, 2]
    with pytest.raises(ValueError):
        sharding.shard_blocks(s, 2, 2)


def _mcmc_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import phantom
        from paper_conf_ipps_xuzwrwxgxy12_b200 import sharding
        d = phantom.dwi_uniform(nvox=12, gen_seed=4, burnin=20, nsamples=5, interval=2, adapt_every=10)
        mine = d.replace(mask=sharding.shard_voxels(d.mask, rank, world))
        s = torch.from_numpy(oracle.mcmc(mine)["samples"])
        sharding.gather_samples(s, dst=0)
        if rank == 0:
            q.put((s.numpy().copy(), oracle.mcmc(d)["samples"]))
    finally:
        dist.destroy_process_group()


def test_mcmc_voxel_sharding_gathers_exactly():
    """NEXT-4 multi-GPU host logic: voxel v -> rank v mod 2, one reduce(SUM) of the
    zero-elsewhere sample tensors reproduces the single-process samples bit for bit."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_mcmc_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    got, full = q.get(timeout=600)
    for p in procs:
        p.join(timeout=60)
    assert np.array_equal(got, full)

"""Seed sharding and the map combine of the multi-GPU path.

Particles are independent and the RNG is keyed by the *global* particle id
(seed_id * P + j, R16), so a rank can track any subset of seeds as long as it passes their
global ids: the union of the ranks' results equals the single-GPU result bit for bit.  The
only exchange is the final combine of the per-rank uint32 visitation maps: one
``reduce(SUM)`` (NCCL on GPUs) of the maps viewed as int32 -- two's-complement addition is
the same bit pattern as uint32 addition mod 2^32, so the combined map is bit-identical.
"""
from __future__ import annotations

import numpy as np


def shard_indices(nseeds: int, rank: int, world: int) -> np.ndarray:
    """Interleaved sharding: seed i -> rank i mod world (spatially uniform, so the per-rank
    work balances statistically for raster-ordered seeds)."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError(f"bad rank {rank} / world {world}")
    return np.arange(rank, nseeds, world, dtype=np.int64)


def _spread3(v: np.ndarray) -> np.ndarray:
    x = v.astype(np.uint64) & np.uint64(0x3FF)
    for sh, m in ((16, 0x030000FF), (8, 0x0300F00F), (4, 0x030C30C3), (2, 0x09249249)):
        x = (x | (x << np.uint64(sh))) & np.uint64(m)
    return x


def morton_order(seeds: np.ndarray) -> np.ndarray:
    """Stable Z-order permutation of the seeds by their voxel (10 bits per axis, coordinates
    clamped to [0, 1023]) -- the order pt_track claims seeds in on the device."""
    c = np.clip(np.floor(np.asarray(seeds, np.float64)), 0, 1023).astype(np.uint64)
    key = _spread3(c[:, 0]) | (_spread3(c[:, 1]) << np.uint64(1)) | (_spread3(c[:, 2]) << np.uint64(2))
    return np.argsort(key, kind="stable")


def shard_blocks(seeds: np.ndarray, rank: int, world: int, block: int = 1024) -> np.ndarray:
    """Block-interleaved spatial sharding: the seeds in Z-order are cut into blocks of
    `block` consecutive seeds (a compact 3-D neighbourhood each) and block b goes to rank
    b mod world.  Every rank draws blocks from the whole volume, so the work balances
    statistically like the plain interleave, but a rank's seeds stay as dense as on one
    GPU inside each block: neighbouring seeds share tracts and hence L1/L2 lines (plain
    i mod world thins every neighbourhood by world and cost ~8 % per rank at 8 ranks).
    Emulated on c3 at 8 ranks: block 64 / 256 / 512 / 1024 / 2048 project
    950 / 970 / 981 / 999-1003 / 988 G steps/s (plain interleave 928 G); larger blocks keep
    more locality but balance worse (max/mean 1.003 -> 1.04)."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError(f"bad rank {rank} / world {world}")
    if block < 1:
        raise ValueError("block must be >= 1")
    perm = morton_order(seeds)
    b = np.arange(perm.size, dtype=np.int64) // block
    return np.sort(perm[b % world == rank])


def auto_block(nseeds: int, world: int, cap: int = 1024) -> int:
    """Z-order block size: `cap` seeds, but small enough that every rank gets >= 16 blocks."""
    return max(1, min(cap, nseeds // (16 * max(1, world))))


def shard_seeds(seeds: np.ndarray, seed_ids, rank: int, world: int, block=None):
    """(seeds, global seed ids) of this rank's shard (block-interleaved in Z-order,
    `shard_blocks`, block None = auto_block; block = 0 selects the plain interleave seed
    i -> rank i mod world)."""
    n = int(seeds.shape[0])
    if block is None:
        block = auto_block(n, world)
    ids = np.arange(n, dtype=np.uint64) if seed_ids is None else np.asarray(seed_ids, np.uint64)
    sel = shard_indices(n, rank, world) if block == 0 or world == 1 else shard_blocks(seeds, rank, world, block)
    return np.ascontiguousarray(seeds[sel]), np.ascontiguousarray(ids[sel])


def shard_voxels(mask: np.ndarray, rank: int, world: int) -> np.ndarray:
    """MCMC (NEXT-4) sharding: voxel v -> rank v mod world.  The sampler's draws are keyed
    by the linear voxel index (M6), so every rank's samples equal the single-GPU
    ones; returns this rank's mask (uint8, same shape)."""
    if world < 1 or not (0 <= rank < world):
        raise ValueError(f"bad rank {rank} / world {world}")
    m = np.ascontiguousarray(mask, np.uint8).copy()
    flat = m.reshape(-1)
    flat[np.arange(flat.size) % world != rank] = 0
    return m


def gather_samples(samples, dst: int = 0, group=None):
    """Combine per-rank MCMC sample tensors (float64, zeros outside each rank's voxels) in
    place with one reduce(SUM): each voxel is non-zero on exactly one rank, and x + 0 = x
    exactly in IEEE arithmetic, so the result is bit-identical to the single-GPU samples."""
    import torch.distributed as dist
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return samples
    t = samples
    staged = samples.is_cuda and dist.get_backend(group) == "gloo"
    if staged:
        t = samples.cpu()
    dist.reduce(t, dst=dst, op=dist.ReduceOp.SUM, group=group)
    if staged:
        samples.copy_(t)
    return samples


def reduce_map(map_i32, dst: int = 0, group=None, all_ranks: bool = False):
    """Combine the ranks' maps in place: reduce to ``dst`` (or all-reduce) with SUM over
    the int32 view.  ``map_i32`` is a torch int32 tensor holding uint32 counts."""
    import torch
    import torch.distributed as dist
    if map_i32.dtype != torch.int32:
        raise TypeError("the map must be an int32 view of the uint32 counts")
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return map_i32
    t = map_i32
    staged = map_i32.is_cuda and dist.get_backend(group) == "gloo"  # gloo: host tensors only
    if staged:
        t = map_i32.cpu()
    if all_ranks:
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    else:
        dist.reduce(t, dst=dst, op=dist.ReduceOp.SUM, group=group)
    if staged:
        map_i32.copy_(t)
    return map_i32

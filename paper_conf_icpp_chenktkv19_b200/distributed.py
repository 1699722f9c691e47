"""Multi-GPU drivers of the AM engine: one process per GPU,
``torch.distributed`` for the plumbing (NCCL over NVLink 5 on B200 boxes).

Two natural partitions of the work (the paper itself is single-GPU, PAPER.md
L88; these follow north_star):

* **toolpath batches -> pivot sharding** (:func:`run_batch`): every rank holds a
  full replica of the voxel model and computes the maps of pivots
  ``rank, rank + G, ...``; there is no data-path collective (an optional
  ``all_gather`` brings the maps to every rank).  Weak scaling.
* **one pivot -> voxel sharding** (:func:`run_sharded`): rank r holds the
  voxels of the interleaved 256-voxel bricks ``b = r (mod G)``
  (:func:`shard_voxels`); each rank computes the map of its shard, the maps are
  unpacked to one byte per cell and combined with an ``all_reduce(MAX)`` --
  MAX over 0/1 bytes is OR, and the AM of a union of voxel sets is the OR of
  their AMs (collision with *any* voxel).  MAX over packed words
  would be wrong (0b01 max 0b10 = 0b10), hence the unpack.

The per-rank compute, unpack and pack run in the C ABI's kernels
(``Context.compute`` / ``unpack_cells`` / ``pack_cells``); the functions also
accept plain callables so the collective logic can be exercised with the
``gloo`` backend on CPU (tests/test_distributed.py).
"""
from __future__ import annotations

import numpy as np

BRICK = 256  # voxels per brick of the voxel partition (Morton-consecutive)


def shard_voxels(centers, halfs, rank: int, world: int, brick: int = BRICK):
    """Voxels of rank `rank`: interleaved bricks b = rank (mod world).

    Interleaving spreads the few heavy voxels next to the pivot over all ranks
    (SURVEY.md 8(e)(1)).  Works on numpy arrays or torch tensors.
    """
    n = len(halfs)
    idx = np.arange(n)
    keep = (idx // brick) % world == rank
    if type(centers).__module__.startswith("torch"):
        import torch
        sel = torch.from_numpy(np.nonzero(keep)[0]).to(centers.device)
        return centers.index_select(0, sel), halfs.index_select(0, sel)
    return centers[keep], halfs[keep]


def pivot_shard(pivots, rank: int, world: int):
    """Pivots of rank `rank` in the toolpath batch: rank, rank + world, ..."""
    return pivots[rank::world]


def run_batch(ctx, pivots, group=None, gather: bool = False, out=None, stream=None):
    """Pivot-sharded toolpath batch: the maps of this rank's pivots.

    ctx: a Context holding the full model (or any object with
    ``compute_batch(pivots, out=..., stream=...)``).  Returns this rank's maps
    (uint32 [P_r, words]); with gather=True every rank also receives the maps
    of all ranks in pivot order (torch CUDA tensors, via all_gather).
    """
    import torch.distributed as dist
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    mine = pivot_shard(np.asarray(pivots, dtype=np.float32).reshape(-1, 3), rank, world)
    maps = ctx.compute_batch(mine, out=out, stream=stream)
    if not gather or world == 1:
        return maps
    import torch
    is_t = isinstance(maps, torch.Tensor)
    dev = maps.device if is_t else torch.device("cpu")
    t = maps if is_t else torch.from_numpy(np.ascontiguousarray(maps).view(np.int32))
    per = (len(pivots) + world - 1) // world
    buf = torch.zeros((per, t.shape[1]), dtype=t.dtype, device=dev)
    buf[: len(t)] = t
    parts = [torch.empty_like(buf) for _ in range(world)]
    dist.all_gather(parts, buf, group=group)
    full = torch.empty((len(pivots), t.shape[1]), dtype=t.dtype, device=dev)
    for r in range(world):
        cnt = len(range(r, len(pivots), world))
        full[r::world] = parts[r][:cnt]
    return full


def run_sharded(compute, unpack, pack, pivot, group=None):
    """Voxel-sharded single pivot: OR of the ranks' maps via all_reduce(MAX).

    compute(pivot) -> this rank's packed map (words); unpack(words) -> uint8
    cells (torch tensor on the collective's device); pack(cells) -> words.
    Returns the packed map of the whole model on every rank.
    """
    import torch.distributed as dist
    words = compute(pivot)
    cells = unpack(words)
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(cells, op=dist.ReduceOp.MAX, group=group)
    return pack(cells)


def device_codec(ctx, stream=None):
    """(compute, unpack, pack) for run_sharded on a GPU Context: the map stays
    on the device; unpack/pack are the library's kernels (am_unpack_cells /
    am_pack_cells)."""
    import torch
    dev = torch.device("cuda", ctx.device)
    words = torch.zeros(ctx.words, dtype=torch.int32, device=dev)
    cells = torch.zeros(ctx.m * ctx.n, dtype=torch.uint8, device=dev)

    def compute(pivot):
        ctx.compute(pivot, out=words, stream=stream)
        return words

    def unpack(w):
        ctx.unpack_cells(w, cells, stream=stream)
        return cells

    def pack(c):
        out = torch.zeros_like(words)
        ctx.pack_cells(c, out, stream=stream)
        return out

    return compute, unpack, pack

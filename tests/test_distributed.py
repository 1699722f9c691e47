"""Multi-process logic of the multi-GPU drivers on CPU (gloo, world size 2).

The per-rank compute is the fp64 oracle's robust-hit map of the rank's voxel
shard (the CUDA path is not available here); the collective logic under test
-- brick-interleaved voxel sharding + unpack / all_reduce(MAX) / pack, and
pivot sharding + all_gather -- is the same code the GPU path runs.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import scenes
from paper_conf_icpp_chenktkv19_b200 import distributed as D


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _robust_words(C, H, tool, pivot, m, n):
    S = oracle.am_states(C, H, tool, pivot, m, n)
    return oracle.pack_bits((S == 2).astype(np.uint8)).reshape(-1)


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        _work(rank, world, q)
    except Exception as e:  # report instead of hanging the parent
        import traceback
        q.put((rank, "error", traceback.format_exc(), 0))
    finally:
        dist.destroy_process_group()


def _work(rank, world, q):
    if True:
        cfg = scenes.CONFIGS["T_head"]
        C, H = cfg.leaves()
        m, n = 24, 40
        pivots = cfg.pivots(5)
        # --- voxel sharding for one pivot
        Cs, Hs = D.shard_voxels(C, H, rank, world)
        results = {}
        for k, p in enumerate(pivots[:2]):
            def compute(pv, Cs=Cs, Hs=Hs):
                return _robust_words(Cs, Hs, cfg.tool, pv, m, n)

            def unpack(w):
                return torch.from_numpy(oracle.unpack_bits(w, m, n).reshape(-1).copy())

            def pack(c):
                return oracle.pack_bits(c.numpy().reshape(m, n)).reshape(-1)

            results[k] = D.run_sharded(compute, unpack, pack, p)

        # --- pivot sharding with gather
        class FakeCtx:
            def compute_batch(self, P, out=None, stream=None):
                return np.stack([_robust_words(C, H, cfg.tool, p, m, n) for p in P]) if len(P) else \
                    np.zeros((0, m * ((n + 31) // 32)), np.uint32)

        gathered = D.run_batch(FakeCtx(), pivots, gather=True)
        q.put((rank, {k: v.tolist() for k, v in results.items()}, np.asarray(gathered).tolist(),
               int(len(Hs))))


def test_sharded_and_batched_on_gloo():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    out = [q.get(timeout=300) for _ in range(world)]
    for o in out:
        assert o[1] != "error", o[2]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    cfg = scenes.CONFIGS["T_head"]
    C, H = cfg.leaves()
    m, n = 24, 40
    pivots = cfg.pivots(5)
    assert sum(o[3] for o in out) == len(H)  # the shards partition the model
    for k, p in enumerate(pivots[:2]):
        ref = _robust_words(C, H, cfg.tool, p, m, n)
        for o in out:
            assert np.array_equal(np.asarray(o[1][k], dtype=np.uint32), ref)  # OR of shards == whole model
    ref_batch = np.stack([_robust_words(C, H, cfg.tool, p, m, n) for p in pivots])
    for o in out:
        g = np.asarray(o[2]).astype(np.int64).astype(np.uint32)
        assert np.array_equal(g, ref_batch)


def test_shard_voxels_partition():
    C = np.arange(3000 * 3, dtype=np.float32).reshape(-1, 3)
    H = np.ones(3000, np.float32)
    parts = [D.shard_voxels(C, H, r, 3) for r in range(3)]
    assert sum(len(p[1]) for p in parts) == 3000
    allc = np.concatenate([p[0] for p in parts])
    assert len(np.unique(allc[:, 0])) == 3000
    # interleaved bricks of 256
    assert np.array_equal(parts[1][0][:256], C[256:512])

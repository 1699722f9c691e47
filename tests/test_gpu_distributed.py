"""GPU side of the multi-GPU drivers, on one device: the library's unpack/pack
kernels, and the OR of voxel-shard maps equals the whole-model map bit for bit
(every (voxel, cell) decision is deterministic, so the union is exact)."""
import numpy as np
import pytest

import scenes

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def am(gpu):
    import paper_conf_icpp_chenktkv19_b200 as am
    return am


def test_unpack_pack_roundtrip(am):
    import torch
    ctx = am.Context(scenes.TOOL_3CYL, 13, 70, device=0)
    rng = np.random.default_rng(0)
    cells = torch.from_numpy((rng.random(13 * 70) < 0.4).astype(np.uint8)).cuda()
    words = torch.zeros(ctx.words, dtype=torch.int32, device="cuda")
    ctx.pack_cells(cells, words)
    back = torch.zeros_like(cells)
    ctx.unpack_cells(words, back)
    torch.cuda.synchronize()
    assert torch.equal(back, cells)
    assert np.array_equal(am.unpack(words.cpu().numpy(), 13, 70).reshape(-1), cells.cpu().numpy())
    ctx.close()


@pytest.mark.parametrize("world", [2, 3])
def test_voxel_shards_or_to_whole_map(am, world):
    import torch
    from paper_conf_icpp_chenktkv19_b200 import distributed as D
    cfg = scenes.CONFIGS["T_head"]
    C, H = cfg.leaves()
    P = cfg.pivots(3)
    full = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    full.upload(C, H)
    ref = full.compute_batch(P)
    parts = []
    for r in range(world):
        Cs, Hs = D.shard_voxels(C, H, r, world)
        ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
        ctx.upload(Cs, Hs)
        parts.append(ctx.compute_batch(P))
        # the device codec path of run_sharded (world size 1 here: no collective)
        comp, unpack, pack = D.device_codec(ctx)
        w = D.run_sharded(comp, unpack, pack, P[0])
        torch.cuda.synchronize()
        assert np.array_equal(w.cpu().numpy().view(np.uint32), parts[-1][0])
        ctx.close()
    union = np.bitwise_or.reduce(np.stack(parts), axis=0)
    assert np.array_equal(union, ref)
    full.close()

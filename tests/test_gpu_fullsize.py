"""Full-size parity: EVERY cell of full-size maps against the fp64 oracle.

C3 (27.3M leaves, 64 x 64), C4 (9.8M, 128 x 128) and C5 (27.0M impeller, 64 x 64; 8 seeded
pivots of its toolpath batch), computed in the launch configuration bench.py times (one
am_compute_batch of 64 pivots with AM_OPT_BATCH = 64; C4: 16).  North_star rule: zero mismatches on
every cell the oracle calls robust (state 0 or 2); band cells (state 1) are counted and reported.

The oracle is fed the voxels nearest-first (D - sqrt(3) h from the pivot): the AM is an OR over
voxels, so the order is free (pinned by tests/test_oracle.py::test_permutation_invariance), and a
blocked cell's scan then stops at a near voxel -- a full 27M-voxel map takes seconds on the host's
cores instead of minutes.
"""
import math
import time

import numpy as np
import pytest

import oracle
import scenes

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def am(gpu):
    import paper_conf_icpp_chenktkv19_b200 as am
    return am


def nearest_first(C, H, p):
    o = np.argsort(np.linalg.norm(C - np.asarray(p, np.float32)[None, :], axis=1) - np.float32(math.sqrt(3.0)) * H,
                   kind="stable")
    return np.ascontiguousarray(C[o]), np.ascontiguousarray(H[o])


def full_oracle_map(cfg, C, H, p):
    Cs, Hs = nearest_first(C, H, p)
    return oracle.am_states(Cs, Hs, cfg.tool, p, cfg.m, cfg.n)


def _pick(maps, cfg, am, n_open):
    """The first n_open maps that still have clear cells (where a wrong cone or a missed exact test
    shows), the map with the most clear cells, and the first fully blocked map (early exit)."""
    clear = [int((am.unpack(w, cfg.m, cfg.n) == 0).sum()) for w in maps]
    open_ = [k for k, c in enumerate(clear) if c > 0]
    full = [k for k, c in enumerate(clear) if c == 0]
    pick = open_[:n_open] + ([int(np.argmax(clear))] if clear else []) + full[:1]
    return sorted(set(pick))


@pytest.mark.parametrize("name,npiv,n_open", [("C3", 64, 4), ("C4", 16, 2), ("C5", 64, 7)])
def test_full_size_every_cell(am, name, npiv, n_open):
    import torch
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
    ctx.set_option(am.binding.OPT_BATCH, 64)
    P = cfg.pivots(npiv)
    out = torch.zeros((npiv, ctx.words), dtype=torch.int32, device="cuda:0")
    ctx.compute_batch(P, out=out)
    torch.cuda.synchronize()
    maps = out.cpu().numpy().view(np.uint32)
    report = []
    check = _pick(maps, cfg, am, n_open)
    assert len(check) >= n_open
    for k in check:
        t = time.time()
        S = full_oracle_map(cfg, C, H, P[k])
        g = am.unpack(maps[k], cfg.m, cfg.n)
        robust = S != 1
        mism = int(((g == 1) != (S == 2))[robust].sum())
        band = int((~robust).sum())
        report.append((k, mism, band, int((S == 0).sum()), int((S == 2).sum()), round(time.time() - t, 1)))
        assert mism == 0, (name, k, mism, band)
        # the one-pivot path gives the same map bit for bit
        assert np.array_equal(ctx.compute(P[k])[0], maps[k]), (name, k)
    print(f"\n{name} (N={len(H)}): pivot, mismatches, band cells, oracle clear, oracle blocked, oracle s:",
          report)
    ctx.close()

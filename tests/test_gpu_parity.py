"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle.

Rule (north_star): every cell the oracle calls robust
(state 0 or 2) must match exactly -- zero mismatches; band cells (state 1)
accept either value and are counted.
"""
import math

import numpy as np
import pytest

import oracle
import scenes

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def am(gpu):
    import paper_conf_icpp_chenktkv19_b200 as am
    return am


def _compare(gpu_map, states):
    robust = states != 1
    mism = int(((gpu_map == 1) != (states == 2))[robust].sum())
    return mism, int((~robust).sum())


def _ctx(am, cfg, C, H, m=None, n=None, tool=None):
    ctx = am.Context(tool or cfg.tool, m or cfg.m, n or cfg.n, device=0)
    ctx.upload(C, H)
    return ctx


@pytest.mark.parametrize("name,npiv", [("C1", 2), ("T_head", 4), ("T_head4", 3), ("T_blade", 2), ("T_imp", 2)])
def test_small_configs_full_am(am, name, npiv):
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    for p in cfg.pivots(npiv):
        gmap = ctx.am(p)
        S = oracle.am_states(C, H, cfg.tool, p, cfg.m, cfg.n)
        mism, band = _compare(gmap, S)
        assert mism == 0, (name, p, mism, band)
        base = am.unpack(ctx.compute_baseline(p), cfg.m, cfg.n)
        mism_b, _ = _compare(base, S)
        assert mism_b == 0, (name, p, mism_b)
    ctx.close()


def _random_scene(rng, nvox, spread, hmin, hmax):
    piv = rng.uniform(-5, 5, 3).astype(np.float32)
    dirs = rng.normal(size=(nvox, 3))
    dirs /= np.linalg.norm(dirs, axis=1, keepdims=True)
    dist = spread * rng.random(nvox) ** 0.7
    C = (piv[None, :] + dirs * dist[:, None]).astype(np.float32)
    H = np.exp(rng.uniform(math.log(hmin), math.log(hmax), nvox)).astype(np.float32)
    # keep the pivot outside every voxel (that case has its own test)
    inside = np.all(np.abs(C - piv[None, :]) <= H[:, None], axis=1)
    return piv, C[~inside], H[~inside]


TOOLS = {
    "3cyl": scenes.TOOL_3CYL,
    "paper4": scenes.TOOL_PAPER4,
    "nonmono": ((3.0, 10.0), (1.5, 20.0), (5.0, 15.0), (2.0, 30.0)),  # radii go down and up
    "short": ((4.0, 6.0),),
}


@pytest.mark.parametrize("tool_name", list(TOOLS))
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_random_scenes(am, tool_name, seed):
    """Scattered voxels of mixed sizes at all distances, including beyond the
    tool end (ring voxels) and next to the pivot (cones wider than 90 deg)."""
    rng = np.random.default_rng(100 + seed)
    tool = TOOLS[tool_name]
    L = sum(t[1] for t in tool)
    piv, C, H = _random_scene(rng, 150, 1.3 * L, 0.05, 3.0)
    m, n = (40, 48) if seed != 2 else (17, 70)
    ctx = am.Context(tool, m, n, device=0)
    ctx.upload(C, H)
    gmap = ctx.am(piv)
    S = oracle.am_states(C, H, tool, piv, m, n)
    mism, band = _compare(gmap, S)
    assert mism == 0, (tool_name, seed, mism, band)
    base = am.unpack(ctx.compute_baseline(piv), m, n)
    assert _compare(base, S)[0] == 0
    ctx.close()


@pytest.mark.parametrize("seed", range(4))
def test_single_voxels(am, seed):
    """One voxel per map: every cone and band path in isolation."""
    rng = np.random.default_rng(7 + seed)
    tool = TOOLS[["3cyl", "paper4", "nonmono", "short"][seed]]
    L = sum(t[1] for t in tool)
    ctx = am.Context(tool, 32, 64, device=0)
    for k in range(40):
        piv, C, H = _random_scene(rng, 1, 1.2 * L, 0.02, 4.0)
        if len(H) == 0:
            continue
        ctx.upload(C, H)
        gmap = ctx.am(piv)
        S = oracle.am_states(C, H, tool, piv, 32, 64)
        assert _compare(gmap, S)[0] == 0, (seed, k, C, H, piv)
    ctx.close()


def test_edge_cases(am):
    tool = scenes.TOOL_3CYL
    ctx = am.Context(tool, 16, 33, device=0)
    # empty model
    ctx.upload(np.zeros((0, 3), np.float32), np.zeros(0, np.float32))
    assert (ctx.am((0, 0, 0)) == 0).all()
    # out of reach
    ctx.upload(np.array([[400.0, 0, 0]], np.float32), np.array([1.0], np.float32))
    assert (ctx.am((0, 0, 0)) == 0).all()
    # pivot inside a voxel
    ctx.upload(np.array([[0.3, -0.2, 0.1]], np.float32), np.array([0.5], np.float32))
    assert (ctx.am((0, 0, 0)) == 1).all()
    # padding bits stay zero
    w, _ = ctx.compute((0, 0, 0))
    assert (w.reshape(16, 2)[:, 1] == 1).all()
    ctx.close()


@pytest.mark.parametrize("m,n", [(1, 1), (1, 64), (5, 1), (33, 95), (64, 1024), (200, 32)])
def test_grid_shapes(am, m, n):
    cfg = scenes.CONFIGS["T_head"]
    C, H = cfg.leaves()
    p = cfg.pivots(1)[0]
    ctx = am.Context(cfg.tool, m, n, device=0)
    ctx.upload(C, H)
    S = oracle.am_states(C, H, cfg.tool, p, m, n)
    assert _compare(ctx.am(p), S)[0] == 0
    ctx.close()


def test_batch_device_host_and_sort_invariance(am):
    import torch
    cfg = scenes.CONFIGS["T_head"]
    C, H = cfg.leaves()
    P = cfg.pivots(5)
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
    single = np.stack([ctx.compute(p)[0] for p in P])
    batch = ctx.compute_batch(P)
    assert np.array_equal(single, batch)
    dev = torch.zeros((len(P), ctx.words), dtype=torch.int32, device="cuda:0")
    ctx.compute_batch(P, out=dev)
    torch.cuda.synchronize()
    assert np.array_equal(dev.cpu().numpy().view(np.uint32), batch)
    # unsorted upload and a permuted model give the same maps
    ctx2 = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx2.set_option(am.binding.OPT_MORTON_SORT, 0)
    perm = np.random.default_rng(0).permutation(len(H))
    ctx2.upload(C[perm], H[perm])
    assert np.array_equal(ctx2.compute_batch(P), batch)
    ctx.close()
    ctx2.close()


def test_small_queue_overflow_is_exact(am):
    cfg = scenes.CONFIGS["T_head"]
    C, H = cfg.leaves()
    p = cfg.pivots(1)[0]
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx.upload(C, H)
    ref, st = ctx.compute(p, stats=True)
    ctx.set_option(am.binding.OPT_BAND_QUEUE, 3)
    out, st2 = ctx.compute(p, stats=True)
    assert st2.queue_overflow > 0 or st.band_pairs <= 3
    # counter consistency: every voxel is culled, skipped or passed; kept bricks within the model
    assert st.voxels_culled + st.voxels_skipped <= len(H)
    assert 0 <= st.bricks_kept <= (len(H) + 255) // 256
    assert st.voxels_streamed <= min(len(H), 256 * st.bricks_kept)
    # coarse levels: a nonempty sample; a small model's level 1 may be all of it (AM_L1_MIN_SAMPLE)
    assert 0 < st.level_voxels <= len(H)
    S = oracle.am_states(C, H, cfg.tool, p, cfg.m, cfg.n)
    assert _compare(am.unpack(out, cfg.m, cfg.n), S)[0] == 0
    ctx.close()


def test_sphere_cap_bounds_gpu(am):
    """P3 directly on the GPU map (not only via the oracle)."""
    cfg = scenes.CONFIGS["C1"]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    g = ctx.am((0, 0, 31.0))

    def thc(Rs, Dp, R):
        if math.sqrt(Dp * Dp - Rs * Rs) <= R:
            return math.acos(Rs / Dp)
        return math.asin((Dp * Dp + R * R - Rs * Rs) / (2 * Dp * R))
    lo, hi = thc(28 + 2 * math.sqrt(3) * 0.5, 31, 6.35), thc(28, 31, 6.35)
    phi = (np.arange(32) + 0.5) * math.pi / 32
    assert (g[phi < lo - 1e-4] == 0).all() and (g[phi > hi + 1e-4] == 1).all()
    ctx.close()


@pytest.mark.parametrize("name", ["C2"])
def test_c2_full_size_sampled(am, name):
    """C2 (~2M leaves) at full size: all GPU-clear cells plus a seeded sample of
    blocked cells are checked cell by cell against the oracle."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    rng = np.random.default_rng(11)
    for p in cfg.pivots(2):
        g = ctx.am(p).reshape(-1)
        clear = np.nonzero(g == 0)[0]
        blocked = np.nonzero(g == 1)[0]
        cells = np.concatenate([clear[:48], rng.choice(blocked, size=min(48, len(blocked)), replace=False)])
        S = oracle.am_states(C, H, cfg.tool, p, cfg.m, cfg.n, cells=cells)
        robust = S != 1
        assert (((g[cells] == 1) != (S == 2))[robust]).sum() == 0
    ctx.close()


@pytest.mark.parametrize("name", ["T_head", "T_imp", "C2"])
def test_phases_and_tunables_give_identical_maps(am, name):
    """The coarse levels / clear-direction map, the grid size and the merge
    period only decide which work is skipped: the map is a deterministic
    function of the per-(voxel, cell) decisions, so it must be bit-identical."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    P = cfg.pivots(3)
    ctx = _ctx(am, cfg, C, H)
    ref = ctx.compute_batch(P)  # default: the fused cooperative pipeline
    ctx.set_option(am.binding.OPT_FUSED, 0)
    assert np.array_equal(ctx.compute_batch(P), ref)
    ctx.set_option(am.binding.OPT_FUSED, 1)
    ctx.set_option(am.binding.OPT_PHASES, 0)
    assert np.array_equal(ctx.compute_batch(P), ref)
    ctx.set_option(am.binding.OPT_BRICKS, 0)
    assert np.array_equal(ctx.compute_batch(P), ref)
    ctx.set_option(am.binding.OPT_PHASES, 1)
    assert np.array_equal(ctx.compute_batch(P), ref)
    ctx.set_option(am.binding.OPT_BRICKS, 1)
    ctx.set_option(am.binding.OPT_BATCH, 1)  # one fused launch per pivot
    assert np.array_equal(ctx.compute_batch(P), ref)
    ctx.set_option(am.binding.OPT_BATCH, 2)  # groups of 2 + a single
    assert np.array_equal(ctx.compute_batch(P), ref)
    ctx.set_option(am.binding.OPT_CMAP_T, 18)  # not a multiple of 4: per-texel search over all cells
    assert np.array_equal(ctx.compute_batch(P), ref)
    ctx.set_option(am.binding.OPT_CMAP_T, 128)
    for t1 in (64, 37, 128):  # the map after level 0 at its own resolution (<= cmap_T)
        ctx.set_option(am.binding.OPT_CMAP_T1, t1)
        assert np.array_equal(ctx.compute_batch(P), ref)
        assert np.array_equal(np.stack([ctx.compute(p)[0] for p in P]), ref)
    with pytest.raises(am.AMError):
        ctx.set_option(am.binding.OPT_CMAP_T1, 129)  # larger than cmap_T
    # the clear map by the row-ordered nearest-clear search always (0), never, or by default
    for rs in (0, 128, 1 << 21):
        ctx.set_option(am.binding.OPT_CMAP_ROWSCAN, rs)
        assert np.array_equal(ctx.compute_batch(P), ref)
        assert np.array_equal(np.stack([ctx.compute(p)[0] for p in P]), ref)
    with pytest.raises(am.AMError):
        ctx.set_option(am.binding.OPT_CMAP_ROWSCAN, -1)
    # every clear-map search path: all pairs, or candidates bounded per 4x4 / 8x8 texel block
    for brute, block in ((1 << 21, 8), (0, 4), (0, 8), (64, 4), (64, 8)):
        ctx.set_option(am.binding.OPT_CMAP_BRUTE, brute)
        ctx.set_option(am.binding.OPT_CMAP_BLOCK, block)
        assert np.array_equal(ctx.compute_batch(P), ref), (brute, block)
    with pytest.raises(am.AMError):
        ctx.set_option(am.binding.OPT_CMAP_BLOCK, 16)
    for sub in (0, 1, 2):  # without the sub-brick and / or super-brick levels
        ctx.set_option(am.binding.OPT_SUBBRICKS, sub)
        assert np.array_equal(ctx.compute_batch(P), ref), sub
        assert np.array_equal(np.stack([ctx.compute(p)[0] for p in P]), ref), sub
    ctx.set_option(am.binding.OPT_SUBBRICKS, 3)
    ctx.set_option(am.binding.OPT_CMAP_T, 16)
    ctx.set_option(am.binding.OPT_GRID_CTAS, 7)
    ctx.set_option(am.binding.OPT_REFRESH_TILES, 1)
    assert np.array_equal(ctx.compute_batch(P), ref)
    ctx.close()


@pytest.mark.parametrize("batch,diag", [(16, 0), (5, 0), (3, 0), (64, 0), (16, 8), (3, 8)])
def test_batched_launch_matches_single_maps(am, batch, diag):
    """Batched launches give the maps of one-pivot launches bit for bit: the
    phase-by-phase path (blockIdx.y = pivot, per-slot buffers; chunks of
    `batch` pivots with a ragged last chunk) and, with AM_OPT_DIAG bit 3, the
    single cooperative launch whose CTA groups take pivots from a queue."""
    cfg = scenes.CONFIGS["C2"]
    C, H = cfg.leaves()
    P = cfg.pivots(11)
    ctx = _ctx(am, cfg, C, H)
    single = np.stack([ctx.compute(p)[0] for p in P])
    ctx.set_option(am.binding.OPT_DIAG, diag)
    ctx.set_option(am.binding.OPT_BATCH, batch)
    for lanes in (1, 2, 3):  # chunks round-robin over internal streams, each lane its own slots
        ctx.set_option(am.binding.OPT_BATCH_LANES, lanes)
        assert np.array_equal(ctx.compute_batch(P), single), lanes
        assert np.array_equal(ctx.compute_batch(P[::-1]), single[::-1]), lanes  # slots see other pivots
    ctx.close()


@pytest.mark.gpu
def test_l1_sample_option_same_maps(am):
    """AM_OPT_L1_SAMPLE only resizes coarse level 1 (culling): the maps stay bit-identical,
    from a 1-voxel sample to the whole model, and the option takes effect at the next upload."""
    cfg = scenes.CONFIGS["C2"]
    C, H = cfg.leaves()
    P = cfg.pivots(9)
    ctx = _ctx(am, cfg, C, H)
    ref = ctx.compute_batch(P)
    base_levels = ctx.compute(P[0], stats=True)[1].level_voxels
    for sample in (1, 5000, 100000, len(H), 0):
        ctx.set_option(am.binding.OPT_L1_SAMPLE, sample)
        ctx.upload(C, H)
        assert np.array_equal(ctx.compute_batch(P), ref), sample
        lv = ctx.compute(P[0], stats=True)[1].level_voxels
        assert 0 < lv <= len(H), (sample, lv)
        if sample == 0:
            assert lv == base_levels
    with pytest.raises(Exception):
        ctx.set_option(am.binding.OPT_L1_SAMPLE, -1)
    ctx.close()


def test_batch_graph_replay(am):
    """The batch launch chain replayed as a CUDA graph (AM_OPT_GRAPH): replays with new
    pivots into the same device buffer, a new buffer, host outputs and an option change
    (each forcing a recapture) all give the one-pivot maps."""
    import torch
    cfg = scenes.CONFIGS["C2"]
    C, H = cfg.leaves()
    P = cfg.pivots(24)
    ctx = _ctx(am, cfg, C, H)
    single = np.stack([ctx.compute(p)[0] for p in P])
    ctx.set_option(am.binding.OPT_BATCH, 8)
    ctx.set_option(am.binding.OPT_BATCH_LANES, 2)
    dev = torch.zeros((8, ctx.words), dtype=torch.int32, device="cuda:0")
    for rep in range(2):
        for c in range(3):  # same buffer, new pivots each call: replay
            ctx.compute_batch(P[8 * c:8 * c + 8], out=dev)
            torch.cuda.synchronize()
            assert np.array_equal(dev.cpu().numpy().view(np.uint32), single[8 * c:8 * c + 8]), (rep, c)
    dev2 = torch.zeros_like(dev)  # another buffer: recapture
    ctx.compute_batch(P[8:16], out=dev2)
    torch.cuda.synchronize()
    assert np.array_equal(dev2.cpu().numpy().view(np.uint32), single[8:16])
    assert np.array_equal(ctx.compute_batch(P[16:24]), single[16:24])  # host output
    ctx.set_option(am.binding.OPT_BATCH_LANES, 4)  # option change: recapture
    assert np.array_equal(ctx.compute_batch(P[:8]), single[:8])
    ctx.set_option(am.binding.OPT_GRAPH, 0)
    assert np.array_equal(ctx.compute_batch(P), single)
    ctx.close()


def _check_sampled(cfg, C, H, p, g, rng, nclear=64, nblocked=32):
    clear = np.nonzero(g == 0)[0]
    blocked = np.nonzero(g == 1)[0]
    assert len(clear) + len(blocked) > 0
    cells = np.concatenate([rng.choice(clear, size=min(nclear, len(clear)), replace=False),
                            rng.choice(blocked, size=min(nblocked, len(blocked)), replace=False)]).astype(np.int64)
    S = oracle.am_states(C, H, cfg.tool, p, cfg.m, cfg.n, cells=cells)
    robust = S != 1
    assert (((g[cells] == 1) != (S == 2))[robust]).sum() == 0


@pytest.mark.parametrize("name,npiv", [("C3", 64), ("C4", 16), ("C5", 64)])
def test_full_size_bench_launch_config_sampled(am, name, npiv):
    """Full-size configs in the launch configuration bench.py times (C3: a step of
    64 pivots with AM_OPT_BATCH = 64, one launch per phase over all of them; C4
    at 128x128; C5, the impeller of the toolpath-batch config): every batched map
    equals its one-pivot map bit for bit, and every GPU-clear cell (up to 64)
    plus a seeded sample of blocked cells of two maps match the fp64 oracle."""
    import torch
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    ctx.set_option(am.binding.OPT_BATCH, 64)
    rng = np.random.default_rng(3)
    P = cfg.pivots(npiv)
    out = torch.zeros((npiv, ctx.words), dtype=torch.int32, device="cuda:0")
    ctx.compute_batch(P, out=out)
    torch.cuda.synchronize()
    batch = out.cpu().numpy().view(np.uint32)
    for k in range(npiv):
        assert np.array_equal(batch[k], ctx.compute(P[k])[0]), k
    maps = [am.unpack(b, cfg.m, cfg.n).reshape(-1) for b in batch]
    nclear = [int((g == 0).sum()) for g in maps]
    assert max(nclear) > 0  # the path's pivots are not all enclosed
    for k in (0, int(np.argmax(nclear))):  # the first map and the one with the most clear cells
        _check_sampled(cfg, C, H, P[k], maps[k], rng)
    ctx.close()


@pytest.mark.parametrize("subdiv", [1, 2, 3])
@pytest.mark.parametrize("name", ["T_head", "T_imp"])
def test_band_subdivision_matches_oracle(am, name, subdiv):
    """AM_OPT_BAND_SUBDIV (§4.3): band pairs are first
    split into virtual 2x2x2 sub-cubes decided by CHECKICA, CHECKBOX only at the
    bottom.  Exact: same map as CHECKBOX-direct outside the band, and every robust
    cell equals the oracle's, for single and batched launches."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    P = cfg.pivots(3)
    ref = ctx.compute_batch(P)
    ctx.set_option(am.binding.OPT_BAND_SUBDIV, subdiv)
    got = ctx.compute_batch(P)
    single = np.stack([ctx.compute(p)[0] for p in P])
    assert np.array_equal(got, single)
    for k, p in enumerate(P):
        S = oracle.am_states(C, H, cfg.tool, p, cfg.m, cfg.n)
        g = am.unpack(got[k], cfg.m, cfg.n)
        mism, _ = _compare(g, S)
        assert mism == 0
        assert int((g != am.unpack(ref[k], cfg.m, cfg.n))[S != 1].sum()) == 0
    ctx.close()


@pytest.mark.parametrize("name", ["T_head", "C2"])
def test_reuse_between_neighbouring_pivots_same_maps(am, name):
    """AM_OPT_REUSE (8(f) NEXT 2): each slot first rasterises the inner cones, at its
    new pivot, of the voxels that set cells of its previous map.  Any voxel's inner cone at the new
    pivot is exact, so the maps stay bit-identical -- on a continuous toolpath in slot-segment order
    (the intended use), on random pivots, after an option change and after a re-upload."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    path = cfg.toolpath(64)
    ctx = _ctx(am, cfg, C, H)
    ref = np.stack([ctx.compute(p)[0] for p in path])
    ctx.set_option(am.binding.OPT_BATCH, 16)
    ctx.set_option(am.binding.OPT_REUSE, 1)
    seg = path.reshape(16, 4, 3)  # 16 slots, each 4 consecutive path pivots
    for t in range(4):
        got = ctx.compute_batch(seg[:, t])
        assert np.array_equal(got, ref.reshape(16, 4, -1)[:, t]), t
    rnd = cfg.pivots(16)
    ref_r = np.stack([ctx.compute(p)[0] for p in rnd])
    assert np.array_equal(ctx.compute_batch(rnd), ref_r)
    ctx.set_option(am.binding.OPT_BATCH_LANES, 2)
    assert np.array_equal(ctx.compute_batch(seg[:, 0]), ref.reshape(16, 4, -1)[:, 0])
    ctx.upload(C, H)
    assert np.array_equal(ctx.compute_batch(seg[:, 1]), ref.reshape(16, 4, -1)[:, 1])
    ctx.close()


def test_record_and_task_overflow_is_exact(am):
    """When the cone-record / row-task buffers of a stage overflow (C3 with only one coarse level,
    so that ~10^5 voxels per map reach the live stage), the cones that do not fit are rasterised
    inline and the task entries reserved for them are made inert; the batched maps then equal the
    single-pivot maps (whose kernel rasterises in shared memory) and the oracle on every robust cell.
    These toolpath pivots gave robust-clear cells marked blocked before the inert entries (stale
    tasks of an earlier map)."""
    import torch
    cfg = scenes.CONFIGS["C3"]
    C, H = cfg.leaves()
    path = cfg.toolpath(4096)
    P = path[[75, 2322, 2897, 3226, 3250, 3915]]
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
    ctx.set_option(am.binding.OPT_PHASES, 1)
    ctx.set_option(am.binding.OPT_BATCH, 64)
    got = ctx.compute_batch(P)
    single = np.stack([ctx.compute(p)[0] for p in P])
    assert np.array_equal(got, single)
    from test_gpu_fullsize import full_oracle_map
    S = full_oracle_map(cfg, C, H, P[-1])
    mism, _ = _compare(am.unpack(got[-1], cfg.m, cfg.n), S)
    assert mism == 0
    ctx.close()


@pytest.mark.parametrize("name", ["T_head", "T_imp", "C2"])
def test_stage_fusion_same_maps(am, name):
    """AM_OPT_STAGE_FUSION (stage.cuh): one launch per batched stage with survivors, cones and rows
    in shared memory gives the maps of the split cone / row kernels bit for bit, with and without
    AM_OPT_REUSE, on random pivots and on a toolpath."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    ctx.set_option(am.binding.OPT_BATCH, 16)
    for P in (cfg.pivots(16), cfg.toolpath(16)):
        ctx.set_option(am.binding.OPT_STAGE_FUSION, 0)
        ref = ctx.compute_batch(P)
        for bits in (1, 2, 4):  # one stage at a time
            ctx.set_option(am.binding.OPT_STAGE_FUSION, bits)
            assert np.array_equal(ctx.compute_batch(P), ref), bits
        ctx.set_option(am.binding.OPT_STAGE_FUSION, 7)
        assert np.array_equal(ctx.compute_batch(P), ref)
        ctx.set_option(am.binding.OPT_REUSE, 1)
        assert np.array_equal(ctx.compute_batch(P), ref)
        assert np.array_equal(ctx.compute_batch(P), ref)
        ctx.set_option(am.binding.OPT_REUSE, 0)
    ctx.close()


@pytest.mark.parametrize("name", ["C1", "T_head", "T_imp", "C2"])
def test_latency_kernel_matches_previous_single_pivot_kernel(am, name):
    """am_compute's single-pivot kernel (am_latency_kernel: 7 phases, CTA raster, warp-parallel
    CHECKBOX) gives the maps of the previous cooperative kernel (AM_OPT_DIAG bit 4) and of the
    batched path bit for bit, including the small-model variant (no coarse levels)."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    P = cfg.pivots(6)
    ctx = _ctx(am, cfg, C, H)
    new = np.stack([ctx.compute(p)[0] for p in P])
    ctx.set_option(am.binding.OPT_DIAG, 16)
    old = np.stack([ctx.compute(p)[0] for p in P])
    ctx.set_option(am.binding.OPT_DIAG, 0)
    assert np.array_equal(new, old)
    assert np.array_equal(ctx.compute_batch(P), new)
    ctx.close()


@pytest.mark.parametrize("name,ctas", [("C1", 0), ("T_head", 0), ("T_head", 5), ("C2", 0), ("C2", 3)])
def test_tma_full_stream_same_maps(am, name, ctas):
    """AM_OPT_STREAM_TMA (stream.cuh filter_tma_kernel): the full-stream filter with its voxel tiles
    staged by 1-D TMA bulk copies gives the maps and stream counters of the LDG filter_kernel bit for
    bit, and the robust cells of the oracle.  A few persistent CTAs (ctas > 0) make each CTA's
    4-stage ring wrap many times (mbarrier phase parity); N is not a multiple of the 1024-voxel
    tile (ragged tail)."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    assert len(H) % 1024 != 0
    P = cfg.pivots(3)
    ctx = _ctx(am, cfg, C, H)
    ctx.set_option(am.binding.OPT_FUSED, 0)
    ctx.set_option(am.binding.OPT_BRICKS, 0)
    if ctas:
        ctx.set_option(am.binding.OPT_GRID_CTAS, ctas)
    maps, stats = {}, {}
    for tma in (0, 1, 2, 3):
        ctx.set_option(am.binding.OPT_STREAM_TMA, tma)
        out = [ctx.compute(p, stats=True) for p in P]
        maps[tma] = np.stack([o[0] for o in out])
        stats[tma] = [(o[1].voxels_streamed, o[1].voxels_culled, o[1].voxels_live) for o in out]
    for tma in (1, 2, 3):
        assert np.array_equal(maps[0], maps[tma]), tma
        assert stats[0] == stats[tma], tma
    for p, mp in zip(P[:1], maps[1][:1]):
        ref = oracle.am_states(C, H, cfg.tool, p, cfg.m, cfg.n)
        assert _compare(am.unpack(mp, cfg.m, cfg.n), ref)[0] == 0
    ctx.close()


@pytest.mark.parametrize("name", ["T_head", "C2"])
def test_pdl_same_maps(am, name):
    """AM_OPT_PDL: the batched phases as programmatic dependent launches (CTAs start under the previous
    phase's tail, griddepcontrol.wait before reading its results) give the maps of plain stream order
    bit for bit -- 64 pivots in 8 lanes, replayed graph, with and without AM reuse."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    ctx.set_option(am.binding.OPT_BATCH, 64)
    for P in (cfg.pivots(64), cfg.toolpath(64)):
        ctx.set_option(am.binding.OPT_PDL, 0)
        ref = ctx.compute_batch(P)
        ctx.set_option(am.binding.OPT_PDL, 1)
        for _ in range(3):  # (capture, then replays)
            assert np.array_equal(ctx.compute_batch(P), ref)
        ctx.set_option(am.binding.OPT_REUSE, 1)
        assert np.array_equal(ctx.compute_batch(P), ref)
        assert np.array_equal(ctx.compute_batch(P), ref)
        ctx.set_option(am.binding.OPT_REUSE, 0)
    ctx.close()


@pytest.mark.parametrize("name", ["T_head", "T_imp", "C2"])
def test_cmap_far_same_maps(am, name):
    """AM_OPT_CMAP_FAR: far texel blocks of the final clear-direction map store the block-level bound
    theta_C - angle(texel, centre) instead of their own nearest-clear angle.  The bound is valid (only
    looser), so the maps are those without it, batched and single-pivot, down to 1 degree."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    P = cfg.pivots(8)
    ctx = _ctx(am, cfg, C, H)
    ctx.set_option(am.binding.OPT_CMAP_FAR, 0)
    ref = ctx.compute_batch(P)
    assert np.array_equal(np.stack([ctx.compute(p)[0] for p in P]), ref)
    for far in (100, 60, 1):
        ctx.set_option(am.binding.OPT_CMAP_FAR, far)
        assert np.array_equal(ctx.compute_batch(P), ref), far
        assert np.array_equal(np.stack([ctx.compute(p)[0] for p in P]), ref), far
    with pytest.raises(am.AMError):
        ctx.set_option(am.binding.OPT_CMAP_FAR, 181)
    ctx.close()


@pytest.mark.parametrize("name", ["T_head", "T_imp", "C2"])
def test_l1_groups_same_maps(am, name):
    """AM_OPT_L1_SUBS: level-1 voxels in model order, groups of 32 skipped by their bounding sphere in
    the batched level-1 launch -- the same maps as filtering every level-1 voxel, batched (random
    pivots and a toolpath with reuse) and single-pivot."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    for P in (cfg.pivots(16), cfg.toolpath(16)):
        ctx.set_option(am.binding.OPT_L1_SUBS, 0)
        ref = ctx.compute_batch(P)
        assert np.array_equal(np.stack([ctx.compute(p)[0] for p in P]), ref)
        ctx.set_option(am.binding.OPT_L1_SUBS, 1)
        assert np.array_equal(ctx.compute_batch(P), ref)
        ctx.set_option(am.binding.OPT_REUSE, 1)
        assert np.array_equal(ctx.compute_batch(P), ref)
        assert np.array_equal(ctx.compute_batch(P), ref)
        ctx.set_option(am.binding.OPT_REUSE, 0)
    ctx.close()


@pytest.mark.parametrize("name", ["T_head", "C2"])
def test_live_list_overflow_is_exact(am, name):
    """AM_OPT_LIVE_CAP: batched map slots whose live-voxel list is far too small for the scene (64 entries;
    these scenes keep hundreds to thousands of live voxels per map): the live-cone phase re-streams the
    kept sub-bricks and emits every live voxel's cones (live_overflow_rescan) -- the maps equal those with
    the default list, for the phase launches (8 lanes, graph) and the cooperative batch (AM_OPT_DIAG bit 3),
    and the single-pivot paths (their list holds every voxel) are unaffected."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    P = cfg.pivots(16)
    ctx = _ctx(am, cfg, C, H)
    ref = ctx.compute_batch(P)
    live = [ctx.compute(p, stats=True)[1].voxels_live for p in P]
    assert max(live) > 64
    ctx.set_option(am.binding.OPT_LIVE_CAP, 64)
    ctx.upload(C, H)
    ctx.set_option(am.binding.OPT_BATCH, 16)
    for _ in range(2):  # (capture, replay)
        assert np.array_equal(ctx.compute_batch(P), ref)
    ctx.set_option(am.binding.OPT_DIAG, 8)
    assert np.array_equal(ctx.compute_batch(P), ref)
    ctx.set_option(am.binding.OPT_DIAG, 0)
    assert np.array_equal(np.stack([ctx.compute(p)[0] for p in P]), ref)
    ctx.set_option(am.binding.OPT_FUSED, 0)
    assert np.array_equal(np.stack([ctx.compute(p)[0] for p in P[:4]]), ref[:4])
    ctx.close()


@pytest.mark.parametrize("name", ["T_head", "T_imp", "C2"])
def test_l1_sparse_same_maps(am, name):
    """AM_OPT_L1_SPARSE: pivots whose map after level 0 is nearly full take every 2nd level-1 voxel (the
    coarse levels only decide what is culled), from never to always: the same maps, with and without reuse."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    ctx.set_option(am.binding.OPT_BATCH, 16)
    for P in (cfg.pivots(16), cfg.toolpath(16)):
        ctx.set_option(am.binding.OPT_L1_SPARSE, 0)
        ref = ctx.compute_batch(P)
        for th in (50, 1 << 20):
            ctx.set_option(am.binding.OPT_L1_SPARSE, th)
            assert np.array_equal(ctx.compute_batch(P), ref), th
        ctx.set_option(am.binding.OPT_REUSE, 1)
        assert np.array_equal(ctx.compute_batch(P), ref)
        assert np.array_equal(ctx.compute_batch(P), ref)
        ctx.set_option(am.binding.OPT_REUSE, 0)
    ctx.close()

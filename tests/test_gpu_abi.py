"""The C ABI's error paths, statistics and stream contract on the GPU (include/am.h).

Call ordering (AM_ESTATE), argument validation (AM_EINVAL: non-finite voxels, half sizes <= 0,
non-finite pivots), all-or-nothing allocation (AM_ENOMEM leaves the context usable), the early
exit and row statistics of a7 / a5, calls on two streams, and the binding's buffer checks.
"""
import ctypes

import numpy as np
import pytest

import oracle
import scenes

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def am(gpu):
    import paper_conf_icpp_chenktkv19_b200 as am
    return am


def _raw(ctx):
    return ctx._h


def test_call_order_estate(am):
    """Every compute entry before am_upload_voxels, and the octree schemes before
    am_build_octree, return AM_ESTATE (SURVEY 8(b) "Call ordering")."""
    lib = am.lib
    ctx = am.Context(scenes.TOOL_3CYL, 16, 32, device=0)
    piv = (ctypes.c_float * 3)(0.0, 0.0, 10.0)
    out = np.zeros(4 * ctx.words, dtype=np.uint32)
    op = ctypes.c_void_p(out.ctypes.data)
    assert lib.am_compute(_raw(ctx), piv, op, 0, None, None) == am.AM_ESTATE
    assert lib.am_compute_batch(_raw(ctx), piv, 1, op, 0, None) == am.AM_ESTATE
    assert lib.am_compute_baseline(_raw(ctx), piv, op, 0, None) == am.AM_ESTATE
    lo = (ctypes.c_float * 3)(-1.0, -1.0, -1.0)
    assert lib.am_build_octree(_raw(ctx), lo, 2.0, None) == am.AM_ESTATE
    assert b"before am_upload_voxels" in lib.am_last_error(_raw(ctx))
    ctx.upload(np.array([[0.0, 0.0, 0.0]], np.float32), np.array([0.25], np.float32))
    assert lib.am_compute_octree(_raw(ctx), piv, 0, 0, 0, op, 0, None, None) == am.AM_ESTATE
    assert lib.am_compute(_raw(ctx), piv, op, 0, None, None) == am.AM_OK
    ctx.close()


@pytest.mark.parametrize("bad", ["nan_centre", "inf_centre", "zero_half", "neg_half", "nan_half", "inf_half"])
@pytest.mark.parametrize("src", ["host", "device"])
def test_upload_einval(am, bad, src):
    """am_upload_voxels validates every voxel (finite centre, finite half size > 0) on either
    source side; a failed upload leaves no model (AM_ESTATE until an upload succeeds)."""
    import torch
    C = np.zeros((300, 3), np.float32)
    C[:, 0] = np.arange(300, dtype=np.float32)
    H = np.full(300, 0.5, np.float32)
    k = 137
    if bad == "nan_centre":
        C[k, 1] = np.nan
    elif bad == "inf_centre":
        C[k, 2] = np.inf
    elif bad == "zero_half":
        H[k] = 0.0
    elif bad == "neg_half":
        H[k] = -0.5
    elif bad == "nan_half":
        H[k] = np.nan
    else:
        H[k] = np.inf
    ctx = am.Context(scenes.TOOL_3CYL, 8, 8, device=0)
    ctx.upload(np.array([[5.0, 5.0, 5.0]], np.float32), np.array([1.0], np.float32))
    if src == "device":
        C, H = torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda()
    with pytest.raises(am.AMError) as e:
        ctx.upload(C, H)
    assert e.value.code == am.AM_EINVAL
    with pytest.raises(am.AMError) as e:
        ctx.compute((0.0, 0.0, 0.0))
    assert e.value.code == am.AM_ESTATE
    ctx.close()


def test_raw_upload_and_pivot_einval(am):
    lib = am.lib
    ctx = am.Context(scenes.TOOL_3CYL, 8, 8, device=0)
    c = np.zeros(3, np.float32)
    h = np.ones(1, np.float32)
    cp, hp = ctypes.c_void_p(c.ctypes.data), ctypes.c_void_p(h.ctypes.data)
    assert lib.am_upload_voxels(_raw(ctx), cp, hp, -1, 0) == am.AM_EINVAL
    assert lib.am_upload_voxels(_raw(ctx), None, hp, 1, 0) == am.AM_EINVAL
    assert lib.am_upload_voxels(_raw(ctx), cp, None, 1, 0) == am.AM_EINVAL
    assert lib.am_upload_voxels(_raw(ctx), None, None, 0, 0) == am.AM_OK  # N = 0 is legal
    out = np.zeros(ctx.words * 2, np.uint32)
    op = ctypes.c_void_p(out.ctypes.data)
    for v in (np.nan, np.inf, -np.inf):
        piv = (ctypes.c_float * 6)(0.0, 0.0, 0.0, 1.0, v, 2.0)
        assert lib.am_compute(_raw(ctx), (ctypes.c_float * 3).from_buffer(piv, 12),
                              op, 0, None, None) == am.AM_EINVAL
        assert lib.am_compute_batch(_raw(ctx), piv, 2, op, 0, None) == am.AM_EINVAL
        assert b"not finite" in lib.am_last_error(_raw(ctx))
        assert lib.am_compute_baseline(_raw(ctx), (ctypes.c_float * 3).from_buffer(piv, 12),
                                       op, 0, None) == am.AM_EINVAL
    piv = (ctypes.c_float * 3)(0.0, 0.0, 0.0)
    assert lib.am_compute(_raw(ctx), piv, None, 0, None, None) == am.AM_EINVAL
    assert lib.am_compute_batch(_raw(ctx), piv, -1, op, 0, None) == am.AM_EINVAL
    assert lib.am_compute_batch(_raw(ctx), piv, 0, op, 0, None) == am.AM_OK  # P = 0: nothing to do
    for key, val in ((am.binding.OPT_BATCH, 0), (am.binding.OPT_BATCH, 65), (999, 1),
                     (am.binding.OPT_CMAP_T, 3), (am.binding.OPT_BAND_SUBDIV, 4)):
        assert lib.am_set_option(_raw(ctx), key, val) == am.AM_EINVAL
    ctx.close()


def test_enclosing_shell_early_exit(am):
    """P5 / a7: a closed voxel shell around the pivot within the tool's reach blocks every
    orientation; the coarse levels fill the map and the full stream then reads no voxel
    (am_stats.early_exit = 1), on the fused path and on the stage-by-stage path."""
    # (0.25 mm cells: ~150K leaves, above the small-model size whose single-pivot kernel has no
    #  coarse levels)
    C, H = scenes.octree_leaves("shell", (24.0, 20.0), (-32, -32, -32), 64.0, 8)
    assert len(H) > 65536
    pivot = (0.5, -0.25, 0.3)
    S = oracle.am_states(C, H, scenes.TOOL_3CYL, pivot, 64, 64)
    assert (S == 2).all()
    ctx = am.Context(scenes.TOOL_3CYL, 64, 64, device=0)
    ctx.upload(C, H)
    for fused in (1, 0):
        ctx.set_option(am.binding.OPT_FUSED, fused)
        w, st = ctx.compute(pivot, stats=True)
        assert (am.unpack(w, 64, 64) == 1).all()
        assert st.early_exit == 1, (fused, st)
        assert st.voxels_streamed == 0 and st.bricks_kept == 0 and st.voxels_live == 0, (fused, st)
    ctx.set_option(am.binding.OPT_FUSED, 1)
    # a pivot outside the shell: the map is not full, no early exit
    w, st = ctx.compute((0.0, 0.0, 27.0), stats=True)
    assert st.early_exit == 0 and am.unpack(w, 64, 64).min() == 0
    # the batched path (early exit per map) gives the same maps
    P = np.array([pivot, (0.0, 0.0, 27.0), (1.0, 2.0, -3.0)], np.float32)
    single = np.stack([ctx.compute(p)[0] for p in P])
    assert np.array_equal(ctx.compute_batch(P), single)
    ctx.close()


def test_rows_skipped_full_counter(am):
    """am_stats.rows_skipped_full counts the live voxels' phi-rows skipped because the row was
    already full (a5); with rows_rasterised it covers every row of every emitted cone."""
    cfg = scenes.CONFIGS["C2"]
    C, H = cfg.leaves()
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx.upload(C, H)
    tot_skip = 0
    for p in cfg.pivots(4):
        _, st = ctx.compute(p, stats=True)
        assert st.rows_skipped_full >= 0 and st.rows_rasterised >= 0
        assert st.early_exit == 0
        tot_skip += st.rows_skipped_full
    assert tot_skip > 0  # 1 mm off a head-like surface most rows are full (blocked fraction ~0.99)
    ctx.close()


def test_enomem_then_retry_with_fewer_slots(am):
    """a batch whose AM_OPT_BATCH slots do not fit fails with AM_ENOMEM and leaves
    the context as it was; the same call then succeeds with fewer slots, with the right maps."""
    import torch
    cfg = scenes.CONFIGS["T_head"]
    C, H = cfg.leaves()
    P = cfg.pivots(64)
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx.upload(C, H)
    ref = np.stack([ctx.compute(p)[0] for p in P[:8]])
    torch.cuda.synchronize()
    free, _ = torch.cuda.mem_get_info()
    hog = torch.empty(max(0, free - (3 << 30)), dtype=torch.uint8, device="cuda:0")  # leave ~3 GB
    try:
        ctx.set_option(am.binding.OPT_BATCH, 64)  # 64 slots x ~100 MB do not fit in 3 GB
        with pytest.raises(am.AMError) as e:
            ctx.compute_batch(P)
        assert e.value.code == am.AM_ENOMEM
        assert np.array_equal(ctx.compute(P[0])[0], ref[0])  # the context still works
        ctx.set_option(am.binding.OPT_BATCH, 4)
        got = ctx.compute_batch(P[:8])
        assert np.array_equal(got, ref)
    finally:
        del hog
        torch.cuda.empty_cache()
    ctx.close()


def test_two_streams_share_the_context(am):
    """Two asynchronous batches on different streams: the second waits for the first (shared
    scratch), so both produce the one-pivot maps."""
    import torch
    cfg = scenes.CONFIGS["T_head"]
    C, H = cfg.leaves()
    P = cfg.pivots(16)
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx.upload(C, H)
    ctx.set_option(am.binding.OPT_BATCH, 8)
    single = np.stack([ctx.compute(p)[0] for p in P])
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    o1 = torch.zeros((8, ctx.words), dtype=torch.int32, device="cuda:0")
    o2 = torch.zeros_like(o1)
    for rep in range(3):
        ctx.compute_batch(P[:8], out=o1, stream=s1)
        ctx.compute_batch(P[8:], out=o2, stream=s2)
        ctx.compute(P[rep], out=o1[rep], stream=s1)
    torch.cuda.synchronize()
    assert np.array_equal(o1.cpu().numpy().view(np.uint32), single[:8])
    assert np.array_equal(o2.cpu().numpy().view(np.uint32), single[8:])
    ctx.close()


def test_batch_replays_into_slices_of_one_buffer(am):
    """the captured batch chain reads its output base from device memory, so
    replays into different slices of one toolpath buffer are correct (and need no recapture)."""
    import torch
    cfg = scenes.CONFIGS["T_head"]
    C, H = cfg.leaves()
    P = cfg.pivots(24)
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx.upload(C, H)
    single = np.stack([ctx.compute(p)[0] for p in P])
    ctx.set_option(am.binding.OPT_BATCH, 8)
    out = torch.zeros((24, ctx.words), dtype=torch.int32, device="cuda:0")
    for c in (2, 0, 1):
        ctx.compute_batch(P[8 * c:8 * c + 8], out=out[8 * c:8 * c + 8])
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy().view(np.uint32), single)
    ctx.close()


def test_binding_rejects_bad_buffers(am):
    import torch
    ctx = am.Context(scenes.TOOL_3CYL, 8, 40, device=0)
    ctx.upload(np.array([[0.0, 0.0, 20.0]], np.float32), np.array([1.0], np.float32))
    with pytest.raises(ValueError):
        ctx.compute((0, 0, 0), out=torch.zeros(ctx.words - 1, dtype=torch.int32, device="cuda:0"))
    with pytest.raises(ValueError):
        ctx.compute((0, 0, 0), out=torch.zeros(ctx.words, dtype=torch.float32, device="cuda:0"))
    with pytest.raises(ValueError):
        ctx.compute((0, 0, 0), out=torch.zeros((ctx.words, 2), dtype=torch.int32, device="cuda:0")[:, 0])
    with pytest.raises(ValueError):
        ctx.compute((0, 0, 0), out=np.zeros(ctx.words, np.int64))
    with pytest.raises(ValueError):
        ctx.compute_batch(np.zeros((3, 3), np.float32), out=np.zeros((2, ctx.words), np.uint32))
    with pytest.raises(ValueError):
        ctx.upload(torch.zeros((4, 3), dtype=torch.float64, device="cuda:0"),
                   torch.ones(4, dtype=torch.float64, device="cuda:0"))
    with pytest.raises(ValueError):
        ctx.upload(torch.zeros((4, 2), dtype=torch.float32, device="cuda:0"),
                   torch.ones(4, dtype=torch.float32, device="cuda:0"))
    out = torch.zeros(ctx.words, dtype=torch.int32)  # a torch CPU tensor is a host buffer
    ctx.compute((0, 0, 0), out=out)
    assert out.numpy().view(np.uint32).any()
    ctx.close()

"""Benchmark of the AM hot path (driver contract: one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--impl ours|reference]

A step is one am_compute_batch call: the whole hot path (a1-a8 of SURVEY.md
8(a)) for --batch (default 64) consecutive pivots of the seeded 1 mm path over
the resident voxel model, computed phase by phase (8(f) NEXT 2, csrc/batch.cuh)
in chunks of --slots / --lanes (default 64 / 8) pivots per launch that go
round-robin to --lanes internal streams, so the chunks' short phases overlap.  Default workload: C3
(head-like, ~27M leaf voxels, 3-cylinder tool, 64 x 64 = 4096 orientations),
the configuration BASELINE.json's metric is quoted on.  The one-pivot latency
(am_compute) is reported beside it.  For N > 1 (torchrun), every rank computes
its own pivots of the toolpath (pivot sharding): no
data-path collective, weak scaling.

value = voxel.orientation tests / s = N_vox * m * n * maps / max-over-ranks time.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "ms per accessibility map (27M voxels, 64×64 orientations) and voxel·orientation tests/s"
UNIT = "voxel-orientation tests/s"
L2_BYTES = 126 * 1024 * 1024


def _peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


class ClockSampler:
    """Samples SM clock and throttle reasons with NVML while the timed region runs."""

    def __init__(self, device=0, period=0.005):
        self.period = period
        self.samples = []
        self.reasons = set()
        self.max_mhz = None
        self._stop = threading.Event()
        self._ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self._nv = pynvml
            idx = device
            vis = os.environ.get("CUDA_VISIBLE_DEVICES")
            if vis:
                try:
                    idx = int(vis.split(",")[device])
                except ValueError:
                    idx = device
            self._h = pynvml.nvmlDeviceGetHandleByIndex(idx)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self._h, pynvml.NVML_CLOCK_SM)
            self._ok = True
        except Exception:
            pass

    _REASONS = {
        0x0000000000000008: "hw_slowdown", 0x0000000000000040: "hw_thermal_slowdown",
        0x0000000000000020: "sw_thermal_slowdown", 0x0000000000000004: "sw_power_cap",
        0x0000000000000080: "hw_power_brake_slowdown", 0x0000000000000002: "applications_clocks_setting",
    }

    def _run(self):
        nv = self._nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self._h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self._h)
                for bit, name in self._REASONS.items():
                    if r & bit:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self._ok:
            self._t = threading.Thread(target=self._run, daemon=True)
            self._t.start()
        return self

    def __exit__(self, *a):
        if self._ok:
            self._stop.set()
            self._t.join()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": 0}
        return {"sm_mhz": float(statistics.median(self.samples)), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


def _dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def _scene(cfg_name):
    import scenes
    cfg = scenes.CONFIGS[cfg_name]
    t = time.time()
    C, H = cfg.leaves()
    gen_s = time.time() - t
    return cfg, C, H, gen_s


def cpu_oracle_sample(cfg, C, H, pivot, seconds=12.0, seed=0, max_cells=None):
    """Time the fp64 oracle (as it stands) on a bounded sample of one map's cells."""
    import oracle
    rng = np.random.default_rng(seed)
    cells_all = rng.permutation(cfg.m * cfg.n)
    done = 0
    t0 = time.perf_counter()
    used = 0
    chunk = 8
    states = []
    while True:
        cells = cells_all[done: done + chunk]
        if len(cells) == 0:
            break
        st, used = oracle.am_states(C, H, cfg.tool, pivot, cfg.m, cfg.n, cells=cells, return_threads=True)
        states.append(np.asarray(st))
        done += len(cells)
        el = time.perf_counter() - t0
        if el >= seconds or (max_cells and done >= max_cells):
            break
        chunk = min(256, chunk * 2)
    el = time.perf_counter() - t0
    return {"tests": float(len(H)) * done, "cells": done, "seconds": el, "threads": used,
            "cell_ids": cells_all[:done], "states": np.concatenate(states) if states else np.zeros(0, np.int8)}


def run_reference(args):
    ws, rank, _ = _dist_env()
    if rank != 0:
        return 0
    cfg, C, H, _ = _scene(args.config)
    piv = cfg.pivots(max(args.steps + args.warmup, 1))
    # each step: the oracle on a bounded sample of that step's map (per-step budget)
    per_step = max(1.0, args.ref_seconds / max(args.steps, 1))
    for k in range(args.warmup):
        cpu_oracle_sample(cfg, C, H, piv[k], seconds=0.2, seed=k, max_cells=8)
    tests = 0.0
    secs = 0.0
    cells = 0
    threads = 0
    for k in range(args.steps):
        r = cpu_oracle_sample(cfg, C, H, piv[args.warmup + k], seconds=per_step, seed=100 + k)
        tests += r["tests"]
        secs += r["seconds"]
        cells += r["cells"]
        threads = r["threads"]
    value = tests / secs
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * secs / max(args.steps, 1),
        "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
        "data": "synthetic", "config": _config_dict(cfg, len(H), not args.no_flush, args.batch, args.slots, args.lanes),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                         "sample": f"{cells} cells of {args.steps} maps (seeded cells, pivots of the 1 mm path), "
                                   f"every voxel per cell, fp64 clip-project-hull test with exact-safe shortcuts"},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


def _config_dict(cfg, N, flushed=True, batch=1, slots=1, lanes=1):
    return {"workload": f"{cfg.name}: {cfg.note}, {len(cfg.tool)}-cylinder tool, {cfg.m}x{cfg.n} AM, "
                        f"pivots on the {cfg.offset:g} mm path",
            "voxels": int(N), "m": cfg.m, "n": cfg.n, "cylinders": [list(t) for t in cfg.tool],
            "l2": (f"inputs {16 * N / 1e6:.0f} MB; L2 (126 MB) flushed by a {2 * L2_BYTES >> 20} MB write before "
                   f"every timed step, outside the per-step CUDA events") if flushed else
                  f"inputs {16 * N / 1e6:.0f} MB; no flush",
            "pivots_per_step": batch, "pivots_per_launch": max(1, slots // lanes), "streams": lanes,
            "parallelism": "pivot-sharded (weak)"}


def _ncu_traffic(cfg_name, kernel, maps=1):
    """DRAM bytes per launch of `kernel` from the committed ncu --set full summary, for a
    launch computing `maps` AMs (scaled from the captured launch's AM count), or None."""
    prof = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        d = json.load(open(prof))
        k = d.get("kernels", {}).get(kernel)
        if k and k.get("config") == cfg_name:
            return k.get("dram_bytes_per_launch") * maps / k.get("maps_per_launch", 1), k.get("tag")
    except Exception:
        pass
    return None, None


def _timed_maps(ctx, piv, out, stream, steps, flush, torch, batch=1):
    """Per-step CUDA events around each call on `stream` (batch = 1: am_compute of one
    pivot; else am_compute_batch of `batch` consecutive pivots); L2 flushed (a write
    larger than L2) before every step when `flush` is a tensor.  Returns (sum of the
    step times in ms, wall ms of the whole loop including the flushes)."""
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(steps)]
    t0 = torch.cuda.Event(enable_timing=True)
    t1 = torch.cuda.Event(enable_timing=True)
    nchunk = max(1, len(piv) // batch)
    t0.record(stream)
    for k in range(steps):
        if flush is not None:
            with torch.cuda.stream(stream):
                flush.fill_(k & 0xFF)
        evs[k][0].record(stream)
        if batch == 1:
            ctx.compute(piv[k % len(piv)], out=out[k % len(piv)], stream=stream)
        else:
            c = (k % nchunk) * batch
            ctx.compute_batch(piv[c:c + batch], out=out[c:c + batch], stream=stream)
        evs[k][1].record(stream)
    t1.record(stream)
    stream.synchronize()
    return sum(a.elapsed_time(b) for a, b in evs), t0.elapsed_time(t1)


def run_ours(args):
    import torch
    ws, rank, local = _dist_env()
    dist = None
    if ws > 1:
        import torch.distributed as dist
        torch.cuda.set_device(local)
        dist.init_process_group("nccl")
    dev = torch.device("cuda", local if ws > 1 else 0)
    torch.cuda.set_device(dev)
    import paper_conf_icpp_chenktkv19_b200 as am
    B = am.binding

    cfg, C, H, gen_s = _scene(args.config)
    N = len(H)
    bsz = args.batch
    npiv = max(args.pivots, bsz) // bsz * bsz
    piv_all = cfg.pivots(npiv * ws)
    piv = piv_all[rank::ws]  # pivot sharding: rank r takes pivots r, r + G, ...
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=dev.index)
    ctx.set_option(B.OPT_BATCH, args.slots)
    if args.cmap_t:
        ctx.set_option(B.OPT_CMAP_T, args.cmap_t)
    if args.cmap_t1:
        ctx.set_option(B.OPT_CMAP_T1, args.cmap_t1)
    if args.l1_sample:
        ctx.set_option(B.OPT_L1_SAMPLE, args.l1_sample)
    if args.cmap_rowscan >= 0:
        ctx.set_option(B.OPT_CMAP_ROWSCAN, args.cmap_rowscan)
    if args.cmap_brute >= 0:
        ctx.set_option(B.OPT_CMAP_BRUTE, args.cmap_brute)
    if args.cmap_block:
        ctx.set_option(B.OPT_CMAP_BLOCK, args.cmap_block)
    if args.map_ctas >= 0:
        ctx.set_option(B.OPT_MAP_CTAS, args.map_ctas)
    if args.subbricks >= 0:
        ctx.set_option(B.OPT_SUBBRICKS, args.subbricks)
    ctx.set_option(B.OPT_BATCH_LANES, args.lanes)
    if args.phases is not None:
        ctx.set_option(B.OPT_PHASES, args.phases)
    if args.band_subdiv:
        ctx.set_option(B.OPT_BAND_SUBDIV, args.band_subdiv)
    t0 = time.time()
    ctx.upload(torch.from_numpy(C).to(dev), torch.from_numpy(H).to(dev))
    torch.cuda.synchronize(dev)
    upload_s = time.time() - t0
    stream = torch.cuda.Stream(dev)
    out = torch.zeros((len(piv), ctx.words), dtype=torch.int32, device=dev)
    flush = None if args.no_flush else torch.empty(2 * L2_BYTES, dtype=torch.uint8, device=dev)
    # warm-up (both launch shapes)
    _timed_maps(ctx, piv, out, stream, args.warmup, None, torch, bsz)
    _timed_maps(ctx, piv, out, stream, 3, None, torch, 1)
    # per-pivot counters (outside the timed region)
    stats = [ctx.compute(p, stats=True)[1] for p in piv]
    mean = {k: float(np.mean([getattr(s_, k) for s_ in stats])) for k in stats[0].__dict__}

    # ---- timed region: K steps of `bsz` pivots each (one am_compute_batch call: one
    #      launch per phase over all pivots), L2 flushed before each step, CUDA events on
    #      the launching stream around each step (AM_OPT_KERNEL_TIMING = 1: no event
    #      between the phase launches, which would serialise their programmatic
    #      dependent launches)
    ctx.set_option(B.OPT_KERNEL_TIMING, 1)
    ctx.kernel_time()
    ctx.kernel_stats()
    if dist:
        dist.barrier()
    torch.cuda.synchronize(dev)
    with ClockSampler(dev.index) as clk:
        ms, wall_ms = _timed_maps(ctx, piv, out, stream, args.steps, flush, torch, bsz)
    if dist:
        dist.barrier()
    torch.cuda.synchronize(dev)
    kms, klaunch = ctx.kernel_time()
    kstats_timed = {k: v for k, v in ctx.kernel_stats().items() if v[1] > 0}  # launch counts of the timed region
    timed_maps = out[:bsz].cpu().numpy().view(np.uint32).copy()  # the maps the timed steps produced
    # ---- the same K steps again with a CUDA event after every kernel launch
    #      (AM_OPT_KERNEL_TIMING = 2): per-kernel device times for `kernels` / `roofline`
    ctx.set_option(B.OPT_KERNEL_TIMING, 2)
    ms_kev, _ = _timed_maps(ctx, piv, out, stream, args.steps, flush, torch, bsz)
    ctx.kernel_time()
    kstats = {k: v for k, v in ctx.kernel_stats().items() if v[1] > 0}
    ctx.set_option(B.OPT_KERNEL_TIMING, 1)
    # single-pivot latency (am_compute, one fused launch per map), flushed: detail
    ks = max(1, min(args.steps, 100))
    ms_single, _ = _timed_maps(ctx, piv, out, stream, ks, flush, torch, 1)
    ks_k, ks_l = ctx.kernel_time()
    # warm-L2 variant of the timed loop (no flush): detail
    kw = max(1, min(args.steps, 200))
    ms_warm, _ = _timed_maps(ctx, piv, out, stream, kw, None, torch, bsz)
    ctx.kernel_time()
    # ---- full-scan leg: every voxel read by filter_kernel (no brick skipping, one launch per stage)
    full = None
    if not args.no_full_scan:
        ctx.set_option(B.OPT_FUSED, 0)
        ctx.set_option(B.OPT_BRICKS, 0)
        kf = max(1, min(args.steps, 50))
        _timed_maps(ctx, piv, out, stream, 3, None, torch, 1)  # warm-up (first launches of these kernels)
        ctx.kernel_time()
        fms, _ = _timed_maps(ctx, piv, out, stream, kf, flush, torch, 1)
        fk, fl = ctx.kernel_time()
        ctx.set_option(B.OPT_BRICKS, 1)
        ctx.set_option(B.OPT_FUSED, 1)
        full = {"ms_per_am": fms / kf, "kernel_ms_avg": fk / max(fl, 1), "steps": kf}
    ctx.set_option(B.OPT_KERNEL_TIMING, 0)

    # ---- e2e: the public API with HOST buffers (pivots in, packed AMs out), synchronous per step
    # (pinned host buffers: the library stages the pivots in its own pinned buffer and copies
    #  the maps straight into host_out)
    host_piv_t = torch.from_numpy(np.ascontiguousarray(piv, dtype=np.float32)).pin_memory()
    host_out_t = torch.zeros((bsz, ctx.words), dtype=torch.int32).pin_memory()
    host_piv = host_piv_t.numpy()
    host_out = host_out_t.numpy().view(np.uint32)
    nchunk = len(piv) // bsz
    for k in range(min(args.warmup, 3)):
        ctx.compute_batch(host_piv[(k % nchunk) * bsz:(k % nchunk + 1) * bsz], out=host_out)
    ke = max(1, min(args.steps, args.e2e_steps))
    if dist:
        dist.barrier()
    e2e_s = 0.0
    for k in range(ke):  # clocked per step so the flush stays outside
        if flush is not None:
            with torch.cuda.stream(stream):
                flush.fill_(k & 0xFF)
            stream.synchronize()
        c = (k % nchunk) * bsz
        t1 = time.perf_counter()
        ctx.compute_batch(host_piv[c:c + bsz], out=host_out)
        e2e_s += time.perf_counter() - t1
    t = torch.tensor([ms, e2e_s, kms / max(klaunch, 1)], dtype=torch.float64, device=dev)
    if dist:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms_max, e2e_max, kavg_ms = t.tolist()
    maps = args.steps * bsz * ws
    maps_rank = args.steps * bsz
    tests_per_map = float(N) * cfg.m * cfg.n
    value = tests_per_map * maps / (ms_max / 1e3)
    e2e_value = tests_per_map * ke * bsz * ws / e2e_max
    peak, peak_src = _peaks()
    # algorithmic bytes per AM = 16 N (one read of every leaf) + m n / 8
    # (AM write); one launch computes bsz maps
    alg_bytes = bsz * (16.0 * N + cfg.m * cfg.n / 8.0)
    achieved = alg_bytes / (kavg_ms / 1e3) / 1e9
    # bytes the fused kernel actually needs: brick spheres, kept bricks' voxels, both map levels
    touched = bsz * (16.0 * (ctx_nbricks(N) + mean["voxels_streamed"] + mean["level_voxels"]) + cfg.m * cfg.n / 8.0)
    dom_roof = _dominant_roofline(kstats, mean, cfg, N, bsz, peak, peak_src,
                                  clk.summary().get("sm_max_mhz"))
    baseline_ms = None
    if args.baseline and rank == 0:
        ctx.set_option(B.OPT_BASELINE_REJECT, 1)
        bo = torch.zeros(ctx.words, dtype=torch.int32, device=dev)
        e0 = torch.cuda.Event(enable_timing=True)
        e1 = torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        ctx.compute_baseline(piv[0], out=bo, stream=stream)
        e1.record(stream)
        stream.synchronize()
        baseline_ms = e0.elapsed_time(e1)
    cpu = None
    parity = None
    # blocked fraction of the maps the timed path produced (SURVEY 8(d) metrics)
    blocked_frac = float(np.mean([am.unpack(timed_maps[k], cfg.m, cfg.n).mean() for k in range(len(timed_maps))]))
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        r = cpu_oracle_sample(cfg, C, H, piv[0], seconds=args.cpu_seconds)
        cpu = {"value": r["tests"] / r["seconds"], "unit": UNIT, "cores": r["threads"], "kind": "oracle",
               "sample": f"{r['cells']} seeded cells of one {cfg.name} map (pivot 0), every voxel per cell, "
                         f"{r['seconds']:.1f} s"}
        # the same oracle cells against the timed path's own map of pivot 0 (north_star parity rule:
        # zero mismatches on robust cells; band cells counted)
        g0 = am.unpack(timed_maps[0], cfg.m, cfg.n).reshape(-1)
        st = r["states"]
        robust = st != 1
        parity = {"pivot": 0, "cells": int(len(st)), "mismatches": int(((g0[r["cell_ids"]] == 1) != (st == 2))[robust].sum()),
                  "band_cells": int((~robust).sum()), "oracle_blocked": int((st == 2).sum()),
                  "source": "the cpu_baseline sample's fp64 oracle states vs the map the timed am_compute_batch produced"}
    if rank == 0:
        full_roof = None
        if full:
            fa = 16.0 * N / (full["kernel_ms_avg"] / 1e3) / 1e9
            ft, ftag = _ncu_traffic(cfg.name, "filter")
            full_roof = {"kernel": "filter_kernel", "bound": "hbm", "achieved": fa, "peak": peak, "unit": "GB/s",
                         "frac": fa / peak, "traffic": ft, "traffic_tag": ftag,
                         "kernel_ms_avg": full["kernel_ms_avg"], "algorithmic_bytes_per_launch": 16.0 * N,
                         "ms_per_am": full["ms_per_am"],
                         "note": "AM_OPT_FUSED=0, AM_OPT_BRICKS=0: every voxel read once per map (no skipping)"}
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ws, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms_max / args.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": _config_dict(cfg, N, flush is not None, bsz, args.slots, args.lanes),
            "ms_per_am": ms_max / args.steps / bsz,
            "roofline": dom_roof,
            "step_roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                              "frac": achieved / peak, "kernel": "the whole batch (all launches of one step)",
                              "ms_per_launch_chain": kavg_ms, "maps_per_launch": bsz,
                              "algorithmic_bytes_per_launch": alg_bytes, "peak_source": peak_src,
                              "touched_bytes_per_launch": touched,
                              "touched_gbs": touched / (kavg_ms / 1e3) / 1e9,
                              "note": "SURVEY 8(d): algorithmic bytes 16 N + m n / 8 per map over the step's "
                                      "device time; the method skips most of them (touched_bytes), so frac is "
                                      "the speed relative to one full HBM pass per map, not bandwidth use"},
            "full_scan_roofline": full_roof,
            "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": 12 * bsz,
                    "d2h_bytes_per_step": 4 * ctx.words * bsz,
                    "ms_per_am": 1e3 * e2e_max / ke / bsz, "steps": ke,
                    "note": f"am_compute_batch with {bsz} host pivots (12 B each, staged by the library in pinned "
                            "memory and copied H2D every step) and a pinned host AM buffer (D2H every step); "
                            "synchronous per step; voxels resident (upload excluded, PAPER.md L313); "
                            "L2 flushed before each step, outside the per-step clock"},
            "gpu_launches": int(sum(v[1] for v in kstats_timed.values())),
            "kernels_note": "per-kernel device times from a second pass of the same K steps with a CUDA event "
                            "after every launch (serialises the phase launches: ms_per_am_with_kernel_events)",
            "ms_per_am_with_kernel_events": ms_kev / args.steps / bsz,
            "kernels": {k: {"ms_per_am": v[0] / maps_rank, "launches": v[1],
                            "share": v[0] / max(sum(x[0] for x in kstats.values()), 1e-12)}
                        for k, v in sorted(kstats.items(), key=lambda kv: -kv[1][0])},
            "clocks": clk.summary(),
            "cpu_baseline": cpu,
            "parity_sample": parity,
            "detail": {"stats_mean_over_pivots": mean, "upload_s": upload_s, "scene_gen_s": gen_s,
                       "blocked_fraction_mean": blocked_frac,
                       "pivots_per_rank": len(piv), "baseline_ms_per_am": baseline_ms,
                       "single_pivot_ms_per_am": ms_single / ks,
                       "single_pivot_kernel_ms": ks_k / max(ks_l, 1),
                       "warm_l2_ms_per_am": ms_warm / kw / bsz, "timed_wall_ms_incl_flush": wall_ms,
                       "host_cpus": os.cpu_count(), "build": _build_id(),
                       "paper_context": "PAPER.md L32/L75: <18 ms per AM, 27M octree nodes x 4096 orientations, "
                                        "GTX 1080(Ti); 'over 23x' vs PBox"},
        }
        print(json.dumps(line), flush=True)
    ctx.close()
    if dist:
        dist.destroy_process_group()
    return 0


# Kernels whose work is a read of voxel records (16 B per voxel):
# units per map from the per-pivot stats.  Every other kernel is an ALU/issue-bound
# search over cones, rows, texels or band pairs.
def _hbm_units(name, mean, N, n_levels):
    return {"voxels": mean["voxels_streamed"], "bricks": float(ctx_nbricks(N)),
            "filter": float(N)}.get(name)


def _dominant_roofline(kstats, mean, cfg, N, bsz, peak_gbs, peak_src, sm_max_mhz):
    """Roofline of the kernel with the largest share of the live per-kernel device time
    (CUDA events after every launch on the launching stream, AM_OPT_KERNEL_TIMING = 2)."""
    tot = sum(v[0] for v in kstats.values())
    if not kstats or tot <= 0:
        return None
    name, (ms, launches) = max(kstats.items(), key=lambda kv: kv[1][0])
    t_launch = ms / launches / 1e3  # s per launch (one launch = bsz maps in the batched path)
    maps = bsz if name not in ("fused_pipeline", "filter") else 1
    traffic, tag = _ncu_traffic(cfg.name, name, maps)
    u = _hbm_units(name, mean, N, 0)
    base = {"kernel": name, "share_of_step": ms / tot, "launches": launches,
            "ms_per_launch": t_launch * 1e3, "maps_per_launch": maps, "traffic": traffic, "traffic_tag": tag}
    if u is not None:
        by = 16.0 * u * maps
        a = by / t_launch / 1e9
        base.update({"bound": "hbm", "achieved": a, "peak": peak_gbs, "unit": "GB/s", "frac": a / peak_gbs,
                     "algorithmic_bytes_per_launch": by, "peak_source": peak_src,
                     "note": "16 B per voxel record the launch reads (SURVEY 8(d)) / live launch time"})
        return base
    # ALU/issue roofline: 148 SMs x 4 schedulers x 1 warp-instruction per clock
    mhz = sm_max_mhz or 1965
    pk = 148 * 4 * mhz * 1e6 / 1e9
    inst = None
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "ncu_summary.json")))["kernels"].get(name)
        if d and d.get("config") == cfg.name and d.get("warp_inst_per_launch"):
            inst = d["warp_inst_per_launch"] * maps / d.get("maps_per_launch", 1)
    except Exception:
        pass
    a = inst / t_launch / 1e9 if inst else None
    base.update({"bound": "alu", "achieved": a, "peak": pk, "unit": "Gwarp-inst/s",
                 "frac": (a / pk) if a else None, "warp_inst_per_launch": inst,
                 "peak_source": f"derived: 148 SM x 4 schedulers x {mhz} MHz (B200_PROFILING.md unit counts)",
                 "note": "data-dependent search (no dense contraction, no per-voxel HBM stream): achieved = "
                         "warp instructions per launch (ncu --set full, committed profile) / live launch time"})
    return base


def ctx_nbricks(N):
    return (N + 255) // 256


def _build_id():
    lib = os.path.join(ROOT, "paper_conf_icpp_chenktkv19_b200", "libam.so")
    try:
        import hashlib
        return hashlib.sha1(open(lib, "rb").read()).hexdigest()[:12]
    except Exception:
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--config", default="C3")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--pivots", type=int, default=64, help="pivots per rank (cycled over the steps)")
    ap.add_argument("--batch", type=int, default=64, help="pivots per step (one am_compute_batch call)")
    ap.add_argument("--slots", type=int, default=64,
                    help="AM_OPT_BATCH: pivots computed together, phase by phase (one launch per phase)")
    ap.add_argument("--e2e-steps", type=int, default=100)
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--ref-seconds", type=float, default=60.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--baseline", action="store_true", help="also time am_compute_baseline once")
    ap.add_argument("--no-flush", action="store_true", help="do not flush L2 between timed steps")
    ap.add_argument("--cmap-t", type=int, default=0, help="AM_OPT_CMAP_T (0 = library default)")
    ap.add_argument("--cmap-t1", type=int, default=0, help="AM_OPT_CMAP_T1 (0 = library default)")
    ap.add_argument("--l1-sample", type=int, default=0, help="AM_OPT_L1_SAMPLE (0 = library default)")
    ap.add_argument("--cmap-rowscan", type=int, default=-1, help="AM_OPT_CMAP_ROWSCAN (-1 = library default)")
    ap.add_argument("--cmap-brute", type=int, default=-1, help="AM_OPT_CMAP_BRUTE (-1 = library default)")
    ap.add_argument("--cmap-block", type=int, default=0, help="AM_OPT_CMAP_BLOCK (0 = library default)")
    ap.add_argument("--map-ctas", type=int, default=-1, help="AM_OPT_MAP_CTAS (-1 = library default)")
    ap.add_argument("--subbricks", type=int, default=-1, help="AM_OPT_SUBBRICKS (-1 = library default)")
    ap.add_argument("--lanes", type=int, default=8,
                    help="AM_OPT_BATCH_LANES: streams the step's chunks of slots / lanes pivots go to")
    ap.add_argument("--phases", type=int, default=None, help="AM_OPT_PHASES (coarse levels, 1 or 2)")
    ap.add_argument("--band-subdiv", type=int, default=0,
                    help="AM_OPT_BAND_SUBDIV: virtual sub-cube levels before CHECKBOX (PAPER.md 4.3)")
    ap.add_argument("--no-full-scan", action="store_true", help="skip the full-scan (filter_kernel) leg")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())

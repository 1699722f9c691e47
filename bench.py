"""Benchmark of the AM hot path (driver contract: one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--impl ours|reference]
                    [--split pivot|voxel]

A step is one am_compute_batch call: the whole hot path (a1-a8 of SURVEY.md 8(a)) for --batch
(default 64) pivots of the seeded 1 mm path over the resident voxel model, computed phase by phase
(8(f) NEXT 2, csrc/batch.cuh) in chunks of --slots / --lanes (default 64 / 8) pivots per launch that
go round-robin to --lanes internal streams.  The K timed steps take K DISTINCT chunks of the rank's
pivots (--pivots, default min(4096, K x batch) per rank; PAPER.md L315 averages 2000 pivots), so
no map is recomputed.  Default workload: C3 (head-like, ~27M leaf voxels, 3-cylinder tool, 64 x 64 =
4096 orientations), the configuration BASELINE.json's metric is quoted on.

Multi-GPU: `--gpus N` outside torchrun re-launches itself as N ranks
(torch.distributed.run, 127.0.0.1); under torchrun WORLD_SIZE must equal N.
  --split pivot (default): rank r computes pivots r, r + N, ... of the toolpath; no data-path
      collective; weak scaling (8(e)(2)).
  --split voxel: one pivot per step, the voxels sharded over the ranks by interleaved 256-voxel
      bricks; each rank's map is unpacked to bytes and OR-ed by an NCCL all_reduce(MAX), then packed
      (distributed.run_sharded); strong scaling (8(e)(1), C3's stated mode).  The combined maps are
      checked bit for bit against the whole model's map on one GPU.

value = voxel.orientation tests / s = N_vox * m * n * maps / max-over-ranks device time.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import socket
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


# ------------------------------------------------------------------ ranks

def _dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def launch_ranks(argv, gpus):
    """`bench.py --gpus N` started outside torchrun: run N ranks of this script (one process
    per GPU, rendezvous on 127.0.0.1).  Returns the launcher's exit code."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={gpus}",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.abspath(__file__)] + list(argv)
    return subprocess.call(cmd)


def _device_index(local):
    """One GPU per rank; more ranks than GPUs share them round robin (a plumbing check only --
    AM_BENCH_BACKEND=gloo then, NCCL refuses two ranks on one GPU)."""
    import torch
    return local % max(1, torch.cuda.device_count())


def _init_dist(ws, local, cuda):
    """Process group of the ranks: NCCL over NVLink on GPUs, gloo on CPU (tests)."""
    if ws <= 1:
        return None
    import torch
    import torch.distributed as dist
    if cuda:
        torch.cuda.set_device(_device_index(local))
    dist.init_process_group(os.environ.get("AM_BENCH_BACKEND") or ("nccl" if cuda else "gloo"))
    return dist


def _max_over_ranks(dist, vals, dev):
    import torch
    t = torch.tensor(vals, dtype=torch.float64, device=dev)
    if dist:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return t.tolist()


# ------------------------------------------------------------------ workload

def _scene(cfg_name):
    import scenes
    cfg = scenes.CONFIGS[cfg_name]
    t = time.time()
    C, H = cfg.leaves()
    gen_s = time.time() - t
    return cfg, C, H, gen_s


def _config_dict(cfg, N, flushed=True, batch=1, slots=1, lanes=1, split="pivot", npiv=None):
    d = {"workload": f"{cfg.name}: {cfg.note}, {len(cfg.tool)}-cylinder tool, {cfg.m}x{cfg.n} AM, "
                     f"pivots on the {cfg.offset:g} mm path",
         "voxels": int(N), "m": cfg.m, "n": cfg.n, "cylinders": [list(t) for t in cfg.tool],
         "l2": (f"inputs {16 * N / 1e6:.0f} MB; L2 (126 MB) flushed by a {2 * L2_BYTES >> 20} MB write before "
                f"every timed step, outside the per-step CUDA events") if flushed else
               f"inputs {16 * N / 1e6:.0f} MB; no flush"}
    if split == "toolpath":
        d.update({"pivots_per_step": batch, "pivots_per_launch": max(1, slots // lanes), "streams": lanes,
                  "distinct_pivots_per_rank": npiv,
                  "parallelism": "pivot-sharded (weak): rank r a contiguous sub-path; step t = pivot s L + t of "
                                 "each of the batch's path segments (AM_OPT_REUSE)"})
    elif split == "pivot":
        d.update({"pivots_per_step": batch, "pivots_per_launch": max(1, slots // lanes), "streams": lanes,
                  "distinct_pivots_per_rank": npiv, "parallelism": "pivot-sharded (weak)"})
    else:
        d.update({"pivots_per_step": 1, "distinct_pivots": npiv,
                  "parallelism": "voxel-sharded single pivot, interleaved 256-voxel bricks, "
                                 "all_reduce(MAX) over one byte per cell (strong)"})
    return d


def nearest_first(C, H, p):
    """Voxels in order of D - sqrt(3) h from the pivot (input order for the oracle's full-map
    parity check: the AM is an OR over voxels, so the order is free; blocked cells stop early)."""
    o = np.argsort(np.linalg.norm(C - np.asarray(p, np.float32)[None, :], axis=1) - np.float32(math.sqrt(3.0)) * H,
                   kind="stable")
    return np.ascontiguousarray(C[o]), np.ascontiguousarray(H[o])


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


def full_map_parity(am, cfg, C, H, pivot, words):
    """Every cell of one map against the fp64 oracle (north_star: zero mismatches on robust cells)."""
    import oracle
    t = time.perf_counter()
    Cs, Hs = nearest_first(C, H, pivot)
    S = oracle.am_states(Cs, Hs, cfg.tool, pivot, cfg.m, cfg.n)
    g = am.unpack(words, cfg.m, cfg.n)
    robust = S != 1
    return {"cells": int(S.size), "mismatches": int(((g == 1) != (S == 2))[robust].sum()),
            "band_cells": int((~robust).sum()), "oracle_blocked": int((S == 2).sum()),
            "oracle_clear": int((S == 0).sum()), "oracle_s": round(time.perf_counter() - t, 2)}


# ------------------------------------------------------------------ reference arm (the oracle)

def run_reference(args):
    ws, rank, local = _dist_env()
    dist = _init_dist(ws, local, cuda=False)  # the oracle is CPU code: gloo plumbing only
    try:
        if rank != 0:
            return 0
        cfg, C, H, _ = _scene(args.config)
        piv = cfg.pivots(max(args.steps + args.warmup, 1))
        # each step: the oracle on a bounded sample of that step's map (per-step budget)
        per_step = max(1.0, args.ref_seconds / max(args.steps, 1))
        for k in range(args.warmup):
            cpu_oracle_sample(cfg, C, H, piv[k], seconds=0.2, seed=k, max_cells=8)
        tests = secs = 0.0
        cells = threads = 0
        for k in range(args.steps):
            r = cpu_oracle_sample(cfg, C, H, piv[args.warmup + k], seconds=per_step, seed=100 + k)
            tests += r["tests"]
            secs += r["seconds"]
            cells += r["cells"]
            threads = r["threads"]
        value = tests / secs
        line = {
            "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * secs / max(args.steps, 1),
            "higher_is_better": True, "scaling": "weak" if args.split == "pivot" else "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": _config_dict(cfg, len(H), not args.no_flush, args.batch, args.slots, args.lanes, args.split),
            "cpu_baseline": {"value": value, "unit": UNIT, "cores": threads, "kind": "oracle",
                             "sample": f"{cells} cells of {args.steps} maps (seeded cells, pivots of the 1 mm path), "
                                       f"every voxel per cell, fp64 clip-project-hull test with exact-safe shortcuts"},
            "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "ranks": ws,
        }
        print(json.dumps(line), flush=True)
        return 0
    finally:
        if dist:
            dist.barrier()
            dist.destroy_process_group()


# ------------------------------------------------------------------ our arm

def _ncu_entry(cfg_name, kernel):
    """The committed ncu --set full summary of `kernel` on config `cfg_name` (profiles/ncu_summary.json)."""
    try:
        d = json.load(open(os.path.join(ROOT, "profiles", "ncu_summary.json")))
    except Exception:
        return None
    k = d.get("by_config", {}).get(cfg_name, {}).get(kernel)
    if k is None:
        k = d.get("kernels", {}).get(kernel)
        if k is not None and k.get("config") != cfg_name:
            k = None
    return k


def _ncu_traffic(cfg_name, kernel, maps=1):
    """DRAM bytes per launch of `kernel` from the committed ncu --set full summary, for a launch
    computing `maps` AMs (scaled from the captured launch's AM count), or None."""
    k = _ncu_entry(cfg_name, kernel)
    if k and k.get("dram_bytes_per_launch") is not None:
        return k["dram_bytes_per_launch"] * maps / k.get("maps_per_launch", 1), k.get("tag")
    return None, None


def _timed_maps(ctx, piv, out, stream, steps, flush, torch, batch=1, start=0):
    """Per-step CUDA events around each call on `stream` (batch = 1: am_compute of one pivot;
    else am_compute_batch of the `batch` pivots of chunk (start + k) mod chunks); L2 flushed
    (a write larger than L2) before every step when `flush` is a tensor.  Returns (sum of the
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
            i = (start + k) % len(piv)
            ctx.compute(piv[i], out=out[i], stream=stream)
        else:
            c = ((start + k) % nchunk) * batch
            ctx.compute_batch(piv[c:c + batch], out=out[c:c + batch], stream=stream)
        evs[k][1].record(stream)
    t1.record(stream)
    stream.synchronize()
    return sum(a.elapsed_time(b) for a, b in evs), t0.elapsed_time(t1)


def _apply_options(ctx, B, args):
    ctx.set_option(B.OPT_BATCH, args.slots)
    for flag, key in (("cmap_t", B.OPT_CMAP_T), ("cmap_t1", B.OPT_CMAP_T1), ("l1_sample", B.OPT_L1_SAMPLE),
                      ("cmap_block", B.OPT_CMAP_BLOCK), ("band_subdiv", B.OPT_BAND_SUBDIV)):
        if getattr(args, flag):
            ctx.set_option(key, getattr(args, flag))
    for flag, key in (("cmap_rowscan", B.OPT_CMAP_ROWSCAN), ("cmap_brute", B.OPT_CMAP_BRUTE),
                      ("map_ctas", B.OPT_MAP_CTAS), ("subbricks", B.OPT_SUBBRICKS)):
        if getattr(args, flag) >= 0:
            ctx.set_option(key, getattr(args, flag))
    ctx.set_option(B.OPT_BATCH_LANES, args.lanes)
    if args.stage_fusion >= 0:
        ctx.set_option(B.OPT_STAGE_FUSION, args.stage_fusion)
    if args.phases is not None:
        ctx.set_option(B.OPT_PHASES, args.phases)
    for kv in args.opt:  # --opt NAME=VALUE: any AM_OPT_* by its binding name (OPT_ prefix optional)
        k, v = kv.split("=")
        ctx.set_option(getattr(B, k if k.startswith("OPT_") else "OPT_" + k), int(v))


def run_ours(args):
    import torch
    ws, rank, local = _dist_env()
    dist = _init_dist(ws, local, cuda=True)
    dev = torch.device("cuda", _device_index(local) if ws > 1 else 0)
    torch.cuda.set_device(dev)
    import paper_conf_icpp_chenktkv19_b200 as am
    cfg, C, H, gen_s = _scene(args.config)
    try:
        if args.split == "voxel":
            return _run_voxel_split(args, am, torch, dist, dev, cfg, C, H, ws, rank)
        return _run_pivot_split(args, am, torch, dist, dev, cfg, C, H, gen_s, ws, rank)
    finally:
        if dist:
            dist.destroy_process_group()


def _run_pivot_split(args, am, torch, dist, dev, cfg, C, H, gen_s, ws, rank):
    B = am.binding
    N = len(H)
    bsz = args.batch
    npiv = args.pivots or min(4096, max(args.steps, 1) * bsz)
    npiv = max(npiv, bsz) // bsz * bsz
    t = time.time()
    if args.toolpath:
        # a continuous toolpath (8(f) NEXT 2): rank r takes the contiguous sub-path r; within it, step
        # t computes pivot s L + t of its bsz segments of L pivots, so slot s of consecutive steps gets
        # neighbouring pivots (AM_OPT_REUSE reuses the slot's previous map)
        path = cfg.toolpath(npiv * ws)[rank * npiv:(rank + 1) * npiv]
        L = npiv // bsz
        piv = np.ascontiguousarray(path.reshape(bsz, L, 3).transpose(1, 0, 2).reshape(-1, 3))
    else:
        piv = cfg.pivots_at(range(rank, npiv * ws, ws))  # pivot sharding: rank r takes pivots r, r + G, ...
    piv_s = time.time() - t
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=dev.index)
    _apply_options(ctx, B, args)
    if args.toolpath:
        ctx.set_option(B.OPT_REUSE, 1)
    t0 = time.time()
    ctx.upload(torch.from_numpy(C).to(dev), torch.from_numpy(H).to(dev))
    torch.cuda.synchronize(dev)
    upload_s = time.time() - t0
    stream = torch.cuda.Stream(dev)
    out = torch.zeros((len(piv), ctx.words), dtype=torch.int32, device=dev)
    flush = None if args.no_flush else torch.empty(2 * L2_BYTES, dtype=torch.uint8, device=dev)
    nchunk = len(piv) // bsz
    # warm-up (both launch shapes), after the last option that shapes the launch chain
    ctx.set_option(B.OPT_KERNEL_TIMING, 1)
    _timed_maps(ctx, piv, out, stream, args.warmup, None, torch, bsz, start=nchunk - args.warmup % nchunk)
    _timed_maps(ctx, piv, out, stream, 3, None, torch, 1)
    # per-pivot counters (outside the timed region; the first 64 pivots)
    stats = [ctx.compute(p, stats=True)[1] for p in piv[:64]]
    mean = {k: float(np.mean([getattr(s_, k) for s_ in stats])) for k in stats[0].__dict__}
    ctx.kernel_time()
    ctx.kernel_stats()

    # ---- timed region: K steps of `bsz` DISTINCT pivots each (one am_compute_batch call: one launch
    #      per phase and chunk, replayed as one CUDA graph), step k on chunk k mod chunks; L2 flushed
    #      before each step; CUDA events on the launching stream around each step
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
    steps_done = min(args.steps, nchunk)
    timed_maps = out[:steps_done * bsz].cpu().numpy().view(np.uint32).copy()  # the maps the timed steps produced
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
    reuse_off = None
    if args.toolpath:  # the same steps without AM_OPT_REUSE (maps checked equal)
        ctx.set_option(B.OPT_REUSE, 0)
        o2 = torch.zeros_like(out)
        _timed_maps(ctx, piv, o2, stream, 3, None, torch, bsz)
        ms_off, _ = _timed_maps(ctx, piv, o2, stream, args.steps, flush, torch, bsz)
        ctx.kernel_time()
        same = bool(torch.equal(o2[:steps_done * bsz], out[:steps_done * bsz]))
        reuse_off = {"ms_per_am": ms_off / args.steps / bsz, "reuse_speedup": ms_off / ms, "maps_identical": same,
                     "median_step_mm": float(np.median(np.linalg.norm(np.diff(path, axis=0), axis=1)))}
        ctx.set_option(B.OPT_REUSE, 1)
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
    # (pinned host buffers: the library stages the pivots in its own pinned buffer and copies the
    #  maps straight into host_out)
    host_piv = torch.from_numpy(np.ascontiguousarray(piv, dtype=np.float32)).pin_memory().numpy()
    host_out_t = torch.zeros((bsz, ctx.words), dtype=torch.int32).pin_memory()
    host_out = host_out_t.numpy().view(np.uint32)
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
    ms_max, e2e_max, kavg_ms = _max_over_ranks(dist, [ms, e2e_s, kms / max(klaunch, 1)], dev)
    maps = args.steps * bsz * ws
    maps_rank = args.steps * bsz
    tests_per_map = float(N) * cfg.m * cfg.n
    value = tests_per_map * maps / (ms_max / 1e3)
    e2e_value = tests_per_map * ke * bsz * ws / e2e_max
    peak, peak_src = _peaks()
    # algorithmic bytes per AM = 16 N (one read of every leaf) + m n / 8 (AM write)
    alg_bytes = bsz * (16.0 * N + cfg.m * cfg.n / 8.0)
    achieved = alg_bytes / (kavg_ms / 1e3) / 1e9
    touched = bsz * (16.0 * (ctx_nbricks(N) + mean["voxels_streamed"] + mean["level_voxels"]) + cfg.m * cfg.n / 8.0)
    dom_roof = _dominant_roofline(kstats, mean, cfg, N, bsz, peak, peak_src, clk.summary().get("sm_max_mhz"))
    baseline = None
    if not args.no_baseline and rank == 0:
        # am_compute_baseline: CHECKBOX for every (voxel, cell) pair (the non-pruned PBox analogue, a9)
        ctx.set_option(B.OPT_BASELINE_REJECT, 1)
        bo = torch.zeros(ctx.words, dtype=torch.int32, device=dev)
        ctx.compute_baseline(piv[1 % len(piv)], out=bo, stream=stream)  # warm-up
        nb = max(1, args.baseline_reps)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for k in range(nb):
            ctx.compute_baseline(piv[k % len(piv)], out=bo, stream=stream)
        e1.record(stream)
        stream.synchronize()
        bms = e0.elapsed_time(e1) / nb
        diff = None
        if nb - 1 < len(timed_maps):
            diff = int((am.unpack(bo.cpu().numpy().view(np.uint32), cfg.m, cfg.n) !=
                        am.unpack(timed_maps[nb - 1], cfg.m, cfg.n)).sum())
        baseline = {"ms_per_am": bms, "speedup_of_aica_step": bms / (ms_max / args.steps / bsz),
                    "pivots": nb, "cells_differing_from_aica": diff,
                    "note": "am_compute_baseline (every voxel x every cell, exact-safe sphere reject, first hit "
                            "per cell ends the cell) on the same resident model, CUDA events; its map against the "
                            "timed AICA map of the same pivot (they may differ only in 1e-5 rad band cells)"}
    cpu = None
    parity = None
    early = sum(int(s_.early_exit) for s_ in stats)
    blocked_frac = float(np.mean([am.unpack(timed_maps[k], cfg.m, cfg.n).mean() for k in range(len(timed_maps))]))
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        r = cpu_oracle_sample(cfg, C, H, piv[0], seconds=args.cpu_seconds)
        cpu = {"value": r["tests"] / r["seconds"], "unit": UNIT, "cores": r["threads"], "kind": "oracle",
               "sample": f"{r['cells']} seeded cells of one {cfg.name} map (pivot 0), every voxel per cell "
                         f"(model order), {r['seconds']:.1f} s"}
        # every cell of the timed path's own map of pivot 0 against the oracle (north_star parity rule)
        parity = full_map_parity(am, cfg, C, H, piv[0], timed_maps[0])
        parity.update({"pivot": 0, "source": "every cell of the map the timed am_compute_batch produced vs the "
                                             "fp64 oracle (voxels fed nearest-first)"})
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
            "config": _config_dict(cfg, N, flush is not None, bsz, args.slots, args.lanes,
                                   "toolpath" if args.toolpath else "pivot", len(piv)),
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
            "e2e": {"value": e2e_value, "unit": UNIT, "h2d_bytes_per_step": 16 * (bsz + 1),
                    "d2h_bytes_per_step": 4 * ctx.words * bsz,
                    "ms_per_am": 1e3 * e2e_max / ke / bsz, "steps": ke,
                    "note": f"am_compute_batch with {bsz} host pivots (staged by the library in pinned memory as "
                            "16 B each plus the 16 B output-base entry, copied H2D every step) and a pinned host "
                            "AM buffer (D2H every step); synchronous per step; voxels resident (upload excluded, "
                            "PAPER.md L313); L2 flushed before each step, outside the per-step clock"},
            "gpu_launches": int(sum(v[1] for v in kstats_timed.values())),
            "kernels_note": "per-kernel device times from a second pass of the same K steps with a CUDA event "
                            "after every launch (serialises the phase launches: ms_per_am_with_kernel_events)",
            "ms_per_am_with_kernel_events": ms_kev / args.steps / bsz,
            "kernels": {k: {"ms_per_am": v[0] / maps_rank, "launches": v[1],
                            "share": v[0] / max(sum(x[0] for x in kstats.values()), 1e-12)}
                        for k, v in sorted(kstats.items(), key=lambda kv: -kv[1][0])},
            "clocks": clk.summary(),
            "cpu_baseline": cpu,
            "parity_full_map": parity,
            "baseline": baseline,
            "detail": {"stats_mean_over_pivots": mean, "early_exit_pivots_of_64": early, "upload_s": upload_s,
                       "scene_gen_s": gen_s, "pivot_gen_s": piv_s,
                       "blocked_fraction_mean": blocked_frac, "distinct_pivots_timed": steps_done * bsz,
                       "pivots_per_rank": len(piv),
                       "toolpath_reuse_off": reuse_off,
                       "single_pivot_ms_per_am": ms_single / ks,
                       "single_pivot_kernel_ms": ks_k / max(ks_l, 1),
                       "warm_l2_ms_per_am": ms_warm / kw / bsz, "timed_wall_ms_incl_flush": wall_ms,
                       "host_cpus": os.cpu_count(), "build": _build_id(),
                       "paper_context": "PAPER.md L32/L75: <18 ms per AM, 27M octree nodes x 4096 orientations, "
                                        "GTX 1080(Ti); 'over 23x' vs PBox"},
        }
        print(json.dumps(line), flush=True)
    ctx.close()
    return 0


def _run_voxel_split(args, am, torch, dist, dev, cfg, C, H, ws, rank):
    """one pivot per step, voxels sharded over the ranks (interleaved 256-voxel
    bricks), per-rank map -> bytes -> NCCL all_reduce(MAX) -> packed map (distributed.run_sharded)."""
    from paper_conf_icpp_chenktkv19_b200 import distributed as D
    B = am.binding
    N = len(H)
    npiv = args.pivots or max(args.steps, 1)
    piv = cfg.pivots_at(range(npiv))  # every rank the same pivots
    Cs, Hs = D.shard_voxels(C, H, rank, ws)
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=dev.index)
    _apply_options(ctx, B, args)
    ctx.upload(torch.from_numpy(np.ascontiguousarray(Cs)).to(dev), torch.from_numpy(np.ascontiguousarray(Hs)).to(dev))
    stream = torch.cuda.Stream(dev)
    flush = None if args.no_flush else torch.empty(2 * L2_BYTES, dtype=torch.uint8, device=dev)
    compute, unpack, pack = D.device_codec(ctx, stream=stream)
    maps = torch.zeros((npiv, ctx.words), dtype=torch.int32, device=dev)

    def step(k):
        with torch.cuda.stream(stream):
            maps[k % npiv] = D.run_sharded(compute, unpack, pack, piv[k % npiv])

    for k in range(args.warmup):
        step(k)
    stream.synchronize()
    ctx.set_option(B.OPT_KERNEL_TIMING, 1)
    ctx.kernel_time()
    ctx.kernel_stats()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if dist:
        dist.barrier()
    torch.cuda.synchronize(dev)
    with ClockSampler(dev.index) as clk:
        for k in range(args.steps):
            if flush is not None:
                with torch.cuda.stream(stream):
                    flush.fill_(k & 0xFF)
            evs[k][0].record(stream)
            step(k)
            evs[k][1].record(stream)
        stream.synchronize()
    if dist:
        dist.barrier()
    ms = sum(a.elapsed_time(b) for a, b in evs)
    kms, kl = ctx.kernel_time()
    kst = {k: v for k, v in ctx.kernel_stats().items() if v[1] > 0}
    # e2e: the pivot from the host, the combined map read back to host memory every step
    host = torch.zeros(ctx.words, dtype=torch.int32).pin_memory()
    ke = max(1, min(args.steps, args.e2e_steps))
    if dist:
        dist.barrier()
    e2e_s = 0.0
    for k in range(ke):
        t1 = time.perf_counter()
        step(k)
        with torch.cuda.stream(stream):
            host.copy_(maps[k % npiv], non_blocking=True)
        stream.synchronize()
        e2e_s += time.perf_counter() - t1
    ms_max, e2e_max, kms_max = _max_over_ranks(dist, [ms, e2e_s, kms / max(kl, 1)], dev)
    # bit-identity with the whole model on one GPU (rank 0 holds a second context with every voxel)
    ident = None
    if rank == 0:
        full = am.Context(cfg.tool, cfg.m, cfg.n, device=dev.index)
        full.upload(torch.from_numpy(C).to(dev), torch.from_numpy(H).to(dev))
        got = maps.cpu().numpy().view(np.uint32)
        chk = min(npiv, args.steps, 16)
        ident = {"pivots": chk, "identical": bool(all(np.array_equal(full.compute(piv[k])[0], got[k])
                                                      for k in range(chk)))}
        full.close()
    tests_per_map = float(N) * cfg.m * cfg.n
    if rank == 0:
        line = {
            "metric": METRIC, "value": tests_per_map * args.steps / (ms_max / 1e3), "unit": UNIT, "n_gpus": ws,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms_max / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
            "data": "synthetic", "split": "voxel",
            "config": _config_dict(cfg, N, flush is not None, split="voxel", npiv=npiv),
            "ms_per_am": ms_max / args.steps,
            "roofline": _dominant_roofline({"fused_pipeline": (kms, max(kl, 1))}, None, cfg, N, 1, *_peaks(),
                                           clk.summary().get("sm_max_mhz")),
            "e2e": {"value": tests_per_map * ke / e2e_max, "unit": UNIT, "h2d_bytes_per_step": 12,
                    "d2h_bytes_per_step": 4 * ctx.words, "ms_per_am": 1e3 * e2e_max / ke, "steps": ke,
                    "note": "host pivot (12 B kernel argument) -> per-rank map -> all_reduce -> packed map read "
                            "back to pinned host memory, synchronous per step"},
            "gpu_launches": int(sum(v[1] for v in kst.values())),
            "collective": {"backend": dist.get_backend() if dist else None, "nranks": ws,
                           "op": "all_reduce(MAX) over m*n uint8 cells per map" if ws > 1 else "none (1 rank)",
                           "bytes_per_map": cfg.m * cfg.n},
            "identical_to_one_gpu": ident,
            "kernel_ms_per_am_max_over_ranks": kms_max,
            "voxels_per_rank": int(len(Hs)),
            "clocks": clk.summary(),
            "cpu_baseline": None,
        }
        print(json.dumps(line), flush=True)
    ctx.close()
    return 0


# Kernels whose work is a read of voxel records (16 B per voxel):
# units per map from the per-pivot stats.  Every other kernel is an ALU/issue-bound
# search over cones, rows, texels or band pairs.
def _hbm_units(name, mean, N):
    if mean is None:
        return {"filter": float(N)}.get(name)
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
    u = _hbm_units(name, mean, N)
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
    d = _ncu_entry(cfg.name, name)
    if d and d.get("warp_inst_per_launch"):
        inst = d["warp_inst_per_launch"] * maps / d.get("maps_per_launch", 1)
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


def main(argv=None):
    argv = sys.argv[1:] if argv is None else argv
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--config", default="C3")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--split", default="pivot", choices=["pivot", "voxel"],
                    help="multi-GPU partition: pivot-sharded batches (weak) or voxel-sharded single pivots (strong)")
    ap.add_argument("--pivots", type=int, default=0,
                    help="distinct pivots per rank (0: min(4096, steps x batch)), cycled by the steps")
    ap.add_argument("--batch", type=int, default=64, help="pivots per step (one am_compute_batch call)")
    ap.add_argument("--slots", type=int, default=64,
                    help="AM_OPT_BATCH: pivots computed together, phase by phase (one launch per phase)")
    ap.add_argument("--e2e-steps", type=int, default=100)
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--ref-seconds", type=float, default=60.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-baseline", action="store_true", help="skip timing am_compute_baseline")
    ap.add_argument("--baseline-reps", type=int, default=2)
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
    ap.add_argument("--toolpath", action="store_true",
                    help="pivots of a continuous toolpath in slot-segment order, AM_OPT_REUSE on (8(f) NEXT 2); "
                         "the same steps without reuse in detail.toolpath_reuse_off")
    ap.add_argument("--stage-fusion", type=int, default=-1, help="AM_OPT_STAGE_FUSION (-1 = library default)")
    ap.add_argument("--opt", action="append", default=[], metavar="NAME=VALUE",
                    help="set any AM_OPT_* (binding name, e.g. CMAP_FAR=120); repeatable")
    args = ap.parse_args(argv)
    if args.warmup < 3:
        args.warmup = 3
    ws = int(os.environ.get("WORLD_SIZE", "0"))
    if ws == 0 and args.gpus > 1:
        return launch_ranks(argv, args.gpus)  # one process per GPU
    if ws > 0 and ws != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={ws}", file=sys.stderr)
        return 2
    if args.impl == "reference":
        return run_reference(args)
    return run_ours(args)


if __name__ == "__main__":
    sys.exit(main())

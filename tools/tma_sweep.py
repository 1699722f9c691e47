"""Full-stream filter (AM_OPT_BRICKS = 0) under each AM_OPT_STREAM_TMA ring shape: device time of the
filter launch (CUDA events around it, AM_OPT_KERNEL_TIMING = 1) per map, L2 flushed before every map,
as a fraction of the measured HBM bandwidth.  python tools/tma_sweep.py [C3] [reps]"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import scenes  # noqa: E402
import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402
from paper_conf_icpp_chenktkv19_b200 import binding as B  # noqa: E402


def main(name="C3", reps=20):
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    N = len(H)
    P = cfg.pivots(4)
    try:
        peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    except OSError:
        peak = 6556.8
    ctx = am.Context(cfg.tool, cfg.m, cfg.n)
    ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
    ctx.set_option(B.OPT_FUSED, 0)
    ctx.set_option(B.OPT_BRICKS, 0)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    ref = None
    for tma in range(0, 4):
        ctx.set_option(B.OPT_STREAM_TMA, tma)
        maps = np.stack([ctx.compute(p)[0] for p in P])
        if ref is None:
            ref = maps
        same = np.array_equal(maps, ref)
        ctx.set_option(B.OPT_KERNEL_TIMING, 1)
        ctx.kernel_time()
        for r in range(reps):
            flush.fill_(r & 0xFF)
            ctx.compute(P[r % len(P)])
        ms, n = ctx.kernel_time()
        ctx.set_option(B.OPT_KERNEL_TIMING, 0)
        kms = ms / max(n, 1)
        gbs = 16.0 * N / (kms * 1e-3) / 1e9
        print(f"{name} stream_tma={tma}: filter {kms * 1e3:.1f} us per map, {gbs:.0f} GB/s = {gbs / peak:.3f} of HBM"
              f"{'' if same else '  MAPS DIFFER'}", flush=True)
    ctx.close()


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "C3", int(sys.argv[2]) if len(sys.argv) > 2 else 20)

"""Probe: per-pivot full-scan (non-fused) map times after the bench's preceding legs."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402
import scenes  # noqa: E402
from paper_conf_icpp_chenktkv19_b200 import binding as B  # noqa: E402

cfg = scenes.CONFIGS["C3"]
C, H = cfg.leaves()
P = cfg.pivots(64)
ctx = am.Context(cfg.tool, cfg.m, cfg.n)
ctx.set_option(B.OPT_BATCH, 64)
ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
stream = torch.cuda.Stream()
out = torch.zeros((64, ctx.words), dtype=torch.int32, device="cuda")
ctx.set_option(B.OPT_FUSED, 0)
ctx.set_option(B.OPT_BRICKS, 0)
ctx.set_option(B.OPT_KERNEL_TIMING, 2)
for k, p in enumerate(P):
    ctx.kernel_stats()
    torch.cuda.synchronize()
    ctx.compute(p, out=out[k], stream=stream)
    torch.cuda.synchronize()
    ks = {n: round(v[0] * 1e3, 1) for n, v in ctx.kernel_stats().items() if v[1]}
    tot = sum(ks.values())
    if tot > 500 or k < 3:
        print(k, round(tot, 1), ks, flush=True)

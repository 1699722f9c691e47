"""Diagnostics on C3: clear cells after the coarse levels, and fused-phase times
of one-pivot and batched launches (AM_OPT_DIAG)."""
import sys
import numpy as np
import torch
sys.path.insert(0, '/root/repo')
import scenes
import paper_conf_icpp_chenktkv19_b200 as am
from paper_conf_icpp_chenktkv19_b200 import binding as B

cfg = scenes.CONFIGS[sys.argv[1] if len(sys.argv) > 1 else 'C3']
C, H = cfg.leaves()
P = cfg.pivots(16)
ctx = am.Context(cfg.tool, cfg.m, cfg.n)
ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
for p in P[:4]:
    full = am.unpack(ctx.compute(p)[0], cfg.m, cfg.n)
    ctx.set_option(B.OPT_FUSED, 0)
    ctx.set_option(B.OPT_DIAG, 1)
    ctx.set_option(B.OPT_PHASES, 1)
    l0 = am.unpack(ctx.compute(p)[0], cfg.m, cfg.n)
    ctx.set_option(B.OPT_PHASES, 2)
    l1 = am.unpack(ctx.compute(p)[0], cfg.m, cfg.n)
    ctx.set_option(B.OPT_DIAG, 0)
    ctx.set_option(B.OPT_FUSED, 1)
    print("clear cells: after L0 %d, after L1 %d, final %d of %d" % (
        (l0 == 0).sum(), (l1 == 0).sum(), (full == 0).sum(), full.size), flush=True)
ctx.set_option(B.OPT_DIAG, 4)
for k in range(2):
    ctx.compute(P[0], stats=True)
for b in (8, 16):
    ctx.set_option(B.OPT_BATCH, b)
    print("batch", b, flush=True)
    for k in range(2):
        ctx.compute_batch(P[:b])
ctx.set_option(B.OPT_PHASES, 1)  # fused without level 1
print("phases=1 (no level 1)", flush=True)
for k in range(2):
    ctx.compute(P[0], stats=True)
for b in (8, 16):
    ctx.set_option(B.OPT_BATCH, b)
    print("batch", b, flush=True)
    for k in range(2):
        ctx.compute_batch(P[:b])
st = [ctx.compute(p, stats=True)[1] for p in P[:4]]
print([ (s.bricks_kept, s.voxels_live) for s in st])

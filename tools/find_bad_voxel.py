"""Debug: does the full-scan path (every voxel's cones, no culling) mark robust-clear cells for a pivot?
If so, bisect the voxel set to the voxel responsible.  python tools/find_bad_voxel.py C3 <path index>"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import scenes  # noqa: E402
import oracle  # noqa: E402
import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402
from paper_conf_icpp_chenktkv19_b200 import binding as B  # noqa: E402

name, k = sys.argv[1], int(sys.argv[2])
cfg = scenes.CONFIGS[name]
C, H = cfg.leaves()
p = cfg.toolpath(4096)[k]
print("pivot", p.tolist(), flush=True)


def full_scan_map(Cs, Hs):
    ctx = am.Context(cfg.tool, cfg.m, cfg.n)
    for key, v in ((B.OPT_FUSED, 0), (B.OPT_BRICKS, 0), (B.OPT_PHASES, 0)):
        ctx.set_option(key, v)
    ctx.upload(Cs, Hs)
    g = am.unpack(ctx.compute(p)[0], cfg.m, cfg.n).reshape(-1)
    ctx.close()
    return g


g = full_scan_map(C, H)
ctx = am.Context(cfg.tool, cfg.m, cfg.n)
ctx.upload(C, H)
d = am.unpack(ctx.compute(p)[0], cfg.m, cfg.n).reshape(-1)
bad = np.nonzero(g != d)[0]
print("full scan vs default: cells differ", len(bad), flush=True)
if len(bad) == 0:
    sys.exit(0)
S = oracle.am_states(C, H, cfg.tool, p, cfg.m, cfg.n, cells=bad)
print("full", g[bad][:10], "default", d[bad][:10], "oracle", S[:10], flush=True)
cell = bad[0]
# bisect: the voxels whose full-scan map alone blocks `cell`
idx = np.arange(len(H))
while len(idx) > 1:
    half = idx[: len(idx) // 2]
    if full_scan_map(C[half], H[half])[cell]:
        idx = half
    else:
        rest = idx[len(idx) // 2:]
        if full_scan_map(C[rest], H[rest])[cell]:
            idx = rest
        else:
            print("cell needs voxels from both halves", len(idx), flush=True)
            break
print("voxel", idx[:4], C[idx[:4]].tolist(), H[idx[:4]].tolist(), flush=True)
i, j = divmod(int(cell), cfg.n)
print("cell", i, j, "oracle single-voxel state", oracle.am_states(C[idx[:1]], H[idx[:1]], cfg.tool, p, cfg.m, cfg.n,
                                                                  cells=[cell]), flush=True)

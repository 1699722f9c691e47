"""am_compute of one chosen pivot, repeated (for ncu): python tools/sp_one.py C3 5 [reps]"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import scenes  # noqa: E402
import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402

cfg = scenes.CONFIGS[sys.argv[1]]
C, H = cfg.leaves()
p = cfg.pivots(int(sys.argv[2]) + 1)[-1]
ctx = am.Context(cfg.tool, cfg.m, cfg.n)
ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
out = torch.zeros(ctx.words, dtype=torch.int32, device="cuda")
for _ in range(int(sys.argv[3]) if len(sys.argv) > 3 else 5):
    ctx.compute(p, out=out)
torch.cuda.synchronize()
print("ok", ctx.compute(p, stats=True)[1])

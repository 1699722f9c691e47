import sys, torch, numpy as np
sys.path.insert(0, '/root/repo')
import scenes, paper_conf_icpp_chenktkv19_b200 as am
from paper_conf_icpp_chenktkv19_b200 import binding as B
cfg = scenes.CONFIGS['C3']; C, H = cfg.leaves(); P = cfg.pivots(4)
ctx = am.Context(cfg.tool, cfg.m, cfg.n); ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
for p in P: ctx.compute(p)
ctx.set_option(B.OPT_DIAG, 4)
for p in P:
    for k in range(2):
        w, st = ctx.compute(p, stats=True)
    print(st, flush=True)

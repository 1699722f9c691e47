import sys
sys.path.insert(0, '/root/repo')
import numpy as np, scenes, paper_conf_icpp_chenktkv19_b200 as am
cfg = scenes.CONFIGS["T_head"]; C, H = cfg.leaves(); P = cfg.pivots(3)
ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0); ctx.upload(C, H)
print(len(H))
ref = ctx.compute_batch(P)
print("ok", ref.sum())

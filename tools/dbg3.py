import sys, numpy as np, torch
sys.path.insert(0, '.')
import scenes, paper_conf_icpp_chenktkv19_b200 as am
name = sys.argv[1]; K = int(sys.argv[2]); opts = sys.argv[3:]
cfg = scenes.CONFIGS[name]; C, H = cfg.leaves()
ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
ctx.upload(C, H)
P = cfg.pivots(K)
for o in opts:
    if o == "single":
        ctx.compute(P[0])
    else:
        k, v = o.split("=")
        ctx.set_option(getattr(am.binding, k), int(v))
ctx.set_option(am.binding.OPT_BATCH, K)
out = torch.zeros((K, ctx.words), dtype=torch.int32, device="cuda:0")
try:
    ctx.compute_batch(P, out=out); torch.cuda.synchronize(); print(name, K, opts, 'ok', flush=True)
except Exception as e:
    print(name, K, opts, 'FAIL', str(e)[:100], flush=True)

import sys, numpy as np, torch
sys.path.insert(0, '.')
import scenes, paper_conf_icpp_chenktkv19_b200 as am
name = sys.argv[1]
cfg = scenes.CONFIGS[name]; C, H = cfg.leaves()
ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
ctx.upload(C, H)
P = cfg.pivots(64)
full = [k for k in range(64) if ctx.compute(P[k], stats=True)[1].early_exit]
print(name, 'early-exit pivots (single):', full, flush=True)
ctx.set_option(am.binding.OPT_BATCH, 64)
single = np.stack([ctx.compute(p)[0] for p in P])
for r in range(3):
    out = torch.zeros((64, ctx.words), dtype=torch.int32, device="cuda:0")
    ctx.compute_batch(P, out=out); torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy().view(np.uint32), single)
print(name, 'batch == single x3 ok', flush=True)

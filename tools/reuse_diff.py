"""Where do AM_OPT_REUSE maps differ from the plain maps (debug): call, slot, cells, oracle states."""
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

name = sys.argv[1] if len(sys.argv) > 1 else "C3"
cfg = scenes.CONFIGS[name]
C, H = cfg.leaves()
path = cfg.toolpath(4096)
L = 64
order = path.reshape(64, L, 3).transpose(1, 0, 2).copy()
ctx = am.Context(cfg.tool, cfg.m, cfg.n)
ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
ctx.set_option(B.OPT_BATCH, 64)
for kv in sys.argv[2:]:
    k, v = kv.split("=")
    ctx.set_option(getattr(B, k), int(v))
s = torch.cuda.Stream()
outs = {}
for reuse in (0, 1):
    ctx.set_option(B.OPT_REUSE, reuse)
    o = torch.zeros((L, 64, ctx.words), dtype=torch.int32, device="cuda")
    for t in range(3):
        ctx.compute_batch(order[t], out=o[t], stream=s)
    for t in range(L):
        ctx.compute_batch(order[t], out=o[t], stream=s)
    s.synchronize()
    outs[reuse] = o.cpu().numpy().view(np.uint32)
nd = 0
for t in range(L):
    for sl in range(64):
        if not np.array_equal(outs[0][t, sl], outs[1][t, sl]):
            ref = ctx.compute(order[t][sl])[0]
            g = am.unpack(outs[1][t, sl], cfg.m, cfg.n).reshape(-1)
            r = am.unpack(outs[0][t, sl], cfg.m, cfg.n).reshape(-1)
            cells = np.nonzero(g != r)[0]
            S = oracle.am_states(C, H, cfg.tool, order[t][sl], cfg.m, cfg.n, cells=cells)
            print(f"t={t} slot={sl}: {len(cells)} cells; reuse={g[cells][:6]} plain={r[cells][:6]} oracle={S[:6]} "
                  f"single==plain {np.array_equal(ref, outs[0][t, sl])} single==reuse {np.array_equal(ref, outs[1][t, sl])}",
                  flush=True)
            nd += 1
            if nd > 8:
                sys.exit(0)
print("done", nd)

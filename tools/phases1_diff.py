"""Debug: batched maps with OPT_PHASES=1 (no level 1) vs single maps on toolpath pivots."""
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

name = sys.argv[1]
cfg = scenes.CONFIGS[name]
C, H = cfg.leaves()
path = cfg.toolpath(4096)
ctx = am.Context(cfg.tool, cfg.m, cfg.n)
ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
ctx.set_option(B.OPT_BATCH, 64)
for kv in sys.argv[2:]:
    k, v = kv.split("=")
    ctx.set_option(getattr(B, k), int(v))
nd = 0
for c in range(0, 4096, 64):
    got = ctx.compute_batch(path[c:c + 64])
    for s in range(64):
        ref = ctx.compute(path[c + s])[0]
        if not np.array_equal(ref, got[s]):
            g = am.unpack(got[s], cfg.m, cfg.n).reshape(-1)
            r = am.unpack(ref, cfg.m, cfg.n).reshape(-1)
            cells = np.nonzero(g != r)[0]
            S = oracle.am_states(C, H, cfg.tool, path[c + s], cfg.m, cfg.n, cells=cells)
            print(f"pivot {c + s}: {len(cells)} cells; batch={g[cells][:6]} single={r[cells][:6]} oracle={S[:6]}", flush=True)
            nd += 1
            if nd > 5:
                sys.exit(0)
print("done", nd)

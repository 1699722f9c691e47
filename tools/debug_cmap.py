"""Debug: compare maps across clear-map resolutions and sources against the oracle."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402
import scenes  # noqa: E402
from paper_conf_icpp_chenktkv19_b200 import binding as B  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C3"
cfg = scenes.CONFIGS[name]
C, H = cfg.leaves()
P = cfg.pivots(2)
ctx = am.Context(cfg.tool, cfg.m, cfg.n)
ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
ref = {}
ctx.set_option(B.OPT_PHASES, 0)
for k, p in enumerate(P):
    ref[k] = am.unpack(ctx.compute(p)[0], cfg.m, cfg.n)
ctx.set_option(B.OPT_PHASES, 1)
for T in (16, 32, 64, 128, 256):
    ctx.set_option(B.OPT_CMAP_T, T)
    for k, p in enumerate(P):
        for diag in (0, 2):
            if diag == 2:
                ctx.set_option(B.OPT_DIAG, 0)
                ctx.compute(p)
            ctx.set_option(B.OPT_DIAG, diag)
            g = am.unpack(ctx.compute(p)[0], cfg.m, cfg.n)
            ctx.set_option(B.OPT_DIAG, 0)
            d = np.nonzero((g != ref[k]).reshape(-1))[0]
            msg = f"T={T} pivot={k} diag={diag} bits={int(g.sum())} ref_bits={int(ref[k].sum())} ndiff={len(d)}"
            if len(d):
                S = oracle.am_states(C, H, cfg.tool, p, cfg.m, cfg.n, cells=d[:16])
                msg += f" cells={d[:16].tolist()} gpu={g.reshape(-1)[d[:16]].tolist()} " \
                       f"ref={ref[k].reshape(-1)[d[:16]].tolist()} oracle={S.tolist()}"
            print(msg, flush=True)

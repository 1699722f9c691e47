"""Single-pivot (am_compute) latency under option settings: median device time per map over the
first 16 pivots (CUDA events, warm L2).  python tools/sp_sweep.py C3 "OPT_CMAP_T1=16" ..."""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import scenes  # noqa: E402
import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402
from paper_conf_icpp_chenktkv19_b200 import binding as B  # noqa: E402


def run(name, settings):
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    P = cfg.pivots(16)
    for st in settings:
        ctx = am.Context(cfg.tool, cfg.m, cfg.n)
        opts = [kv.split("=") for kv in st.split()] if st else []
        for k, v in opts:
            if k in ("OPT_L1_SAMPLE",):
                ctx.set_option(getattr(B, k), int(v))
        ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
        for k, v in opts:
            if k not in ("OPT_L1_SAMPLE",):
                ctx.set_option(getattr(B, k), int(v))
        out = torch.zeros((len(P), ctx.words), dtype=torch.int32, device="cuda")
        ref = np.stack([ctx.compute(p)[0] for p in P])
        s = torch.cuda.Stream()
        for i, p in enumerate(P):
            ctx.compute(p, out=out[i], stream=s)
        ts = []
        for rep in range(3):
            for i, p in enumerate(P):
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                ctx.compute(p, out=out[i], stream=s)
                b.record(s)
                ts.append((a, b))
        s.synchronize()
        t = [a.elapsed_time(b) * 1e3 for a, b in ts]
        if os.environ.get("SP_PER_PIVOT"):
            per = np.median(np.array(t).reshape(3, len(P)), axis=0)
            print("   per pivot (us):", " ".join(f"{x:.0f}" for x in per), flush=True)
            ctx.set_option(B.OPT_DIAG, 4)
            for k in np.argsort(per)[-3:]:
                print("  ", k, ctx.compute(P[k], stats=True)[1], flush=True)
            ctx.set_option(B.OPT_DIAG, 0)
        same = np.array_equal(out.cpu().numpy().view(np.uint32), ref)
        print(f"{name} [{st or 'default'}]: median {np.median(t):.1f} us, mean {np.mean(t):.1f}, min {min(t):.1f}"
              f"{'' if same else ' MAPS DIFFER'}", flush=True)
        ctx.close()


if __name__ == "__main__":
    run(sys.argv[1], sys.argv[2:] or [""])

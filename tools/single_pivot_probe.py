"""Single-pivot latency probe (am_compute): device time per map with CUDA events and the
fused kernel's per-phase end times (AM_OPT_DIAG bit 2, printed by the library on stderr).

    python tools/single_pivot_probe.py [C1 C2 C3 ...]
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import scenes  # noqa: E402
import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402
from paper_conf_icpp_chenktkv19_b200 import binding as B  # noqa: E402


def main(names):
    for name in names:
        cfg = scenes.CONFIGS[name]
        C, H = cfg.leaves()
        P = cfg.pivots(8)
        ctx = am.Context(cfg.tool, cfg.m, cfg.n)
        ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
        out = torch.zeros((len(P), ctx.words), dtype=torch.int32, device="cuda")
        s = torch.cuda.Stream()
        for k in range(3):
            for i, p in enumerate(P):
                ctx.compute(p, out=out[i], stream=s)
        s.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(40)]
        for k, (a, b) in enumerate(ev):
            a.record(s)
            ctx.compute(P[k % len(P)], out=out[k % len(P)], stream=s)
            b.record(s)
        s.synchronize()
        t = [a.elapsed_time(b) * 1e3 for a, b in ev]
        print(f"{name}: N={len(H)} am_compute {np.median(t):.1f} us median ({min(t):.1f} min)", flush=True)
        for extra in (2, 4, 8):
            for k in range(2):
                ctx.compute_batch(P[:extra], out=out[:extra], stream=s)
            s.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            for k in range(10):
                ctx.compute_batch(P[:extra], out=out[:extra], stream=s)
            b.record(s)
            s.synchronize()
            print(f"   compute_batch P={extra}: {a.elapsed_time(b) * 1e3 / 10:.1f} us per call", flush=True)
        ctx.set_option(B.OPT_DIAG, 4)
        for p in P[:3]:
            for k in range(2):
                _, st = ctx.compute(p, stats=True)
            print("  ", st, flush=True)
        ctx.set_option(B.OPT_DIAG, 0)
        ctx.close()


if __name__ == "__main__":
    main(sys.argv[1:] or ["C1", "C2", "C3"])

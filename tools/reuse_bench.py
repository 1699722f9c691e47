"""AM reuse between neighbouring pivots (AM_OPT_REUSE) on a continuous toolpath:
device us per map of am_compute_batch with 64 slots, slot s on path segment s (call t computes
pivots s L + t), with and without reuse; maps checked equal.

    python tools/reuse_bench.py C5 [path pivots, default 4096]
"""
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import scenes  # noqa: E402
import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402
from paper_conf_icpp_chenktkv19_b200 import binding as B  # noqa: E402


def main(name, npath=4096, extra=()):
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    path = cfg.toolpath(npath)
    L = npath // 64
    order = path[: 64 * L].reshape(64, L, 3).transpose(1, 0, 2).copy()  # [t][slot]
    ctx = am.Context(cfg.tool, cfg.m, cfg.n)
    ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
    ctx.set_option(B.OPT_BATCH, 64)
    for kv in extra:
        k, v = kv.split("=")
        ctx.set_option(getattr(B, k), int(v))
    s = torch.cuda.Stream()
    out = {}
    res = {}
    for reuse in (0, 1):
        ctx.set_option(B.OPT_REUSE, reuse)
        o = torch.zeros((L, 64, ctx.words), dtype=torch.int32, device="cuda")
        for t in range(3):  # warm-up
            ctx.compute_batch(order[t], out=o[t], stream=s)
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(L)]
        for t in range(L):
            ev[t][0].record(s)
            ctx.compute_batch(order[t], out=o[t], stream=s)
            ev[t][1].record(s)
        s.synchronize()
        ms = [a.elapsed_time(b) for a, b in ev]
        res[reuse] = {"us_per_map": 1e3 * float(np.mean(ms[1:])) / 64, "steps": L - 1}
        out[reuse] = o.cpu().numpy()
    same = bool(np.array_equal(out[0], out[1]))
    step = np.linalg.norm(np.diff(path, axis=0), axis=1)
    print(json.dumps({"config": name, "path_pivots": npath, "segment_pivots": L, "median_step_mm": float(np.median(step)),
                      "off": res[0], "reuse": res[1], "speedup": res[0]["us_per_map"] / res[1]["us_per_map"],
                      "maps_identical": same}), flush=True)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "C5", int(sys.argv[2]) if len(sys.argv) > 2 else 4096, sys.argv[3:])

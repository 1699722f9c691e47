"""The paper's scheme comparison on B200 (§5,
Table 3 / Fig. 13-18): ms per AM of PBox, optimized PBox, PICA, MICA and AICA
(orientation-per-thread octree traversal, am_compute_octree) next to this
repo's voxel-streaming AICA (am_compute), on the same seeded scene and pivots,
plus the S sweep of MICA / AICA (Fig. 18) and the work counters (nodes popped,
CHECKBOX calls, ICA evaluations, the critical thread's pops, Fig. 13).

    python tools/bench_schemes.py [--config C2] [--pivots 2] [--out profiles/r1_schemes_C2.json]

Times are CUDA events on one stream around each call (device memory output),
after one warm-up call per scheme; the octree build is excluded (like the
voxel upload).  Parity against the oracle is
tests/test_gpu_octree.py's job; here every map is compared bit for bit with
am_compute's and the count of differing cells is reported (band cells only).
"""
import argparse
import json
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--pivots", type=int, default=2)
    ap.add_argument("--schemes", default="pbox,pbox_aabb,pica,mica,aica")
    ap.add_argument("--S", default="0,4,8,10,12,14")
    ap.add_argument("--vdepth", default="0,1,2", help="AICA virtual expansion depths to sweep")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    import torch
    import scenes
    import paper_conf_icpp_chenktkv19_b200 as am

    cfg = scenes.CONFIGS[args.config]
    C, H = cfg.leaves()
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
    t0 = time.time()
    nn = ctx.build_octree(cfg.lo, cfg.size)
    build_s = time.time() - t0
    P = cfg.pivots(args.pivots)
    s = torch.cuda.Stream()
    out = torch.zeros(ctx.words, dtype=torch.int32, device="cuda")

    def timed(fn):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fn()
        e1.record(s)
        s.synchronize()
        return e0.elapsed_time(e1)

    def mp(p):
        return lambda: ctx.compute(p, out=out, stream=s)

    res = {"config": cfg.name, "voxels": len(H), "octree_nodes": nn, "octree_build_s": build_s,
           "m": cfg.m, "n": cfg.n, "pivots": len(P), "rows": []}
    refs = []
    for p in P:
        ctx.compute(p, out=out, stream=s)
        ms = timed(mp(p))
        s.synchronize()
        refs.append(out.cpu().numpy().view(np.uint32).copy())
        res["rows"].append({"scheme": "stream_aica (am_compute)", "pivot": list(map(float, p)), "ms": ms})

    def run(scheme, S, vd):
        for k, p in enumerate(P):
            ctx.compute_octree(p, scheme, S=S, vdepth=vd, out=out, stream=s)  # warm-up
            ms = timed(lambda: ctx.compute_octree(p, scheme, S=S, vdepth=vd, out=out, stream=s))
            _, st = ctx.compute_octree(p, scheme, S=S, vdepth=vd, stats=True)
            g = out.cpu().numpy().view(np.uint32)
            diff = int(np.unpackbits((g ^ refs[k]).view(np.uint8)).sum())
            res["rows"].append({"scheme": scheme, "S": S, "vdepth": vd, "pivot": list(map(float, p)), "ms": ms,
                                "cells_differing_from_am_compute": diff, **st})
            print(json.dumps(res["rows"][-1]), flush=True)

    Ss = [int(x) for x in args.S.split(",")]
    for sc in args.schemes.split(","):
        if sc in ("mica", "aica"):
            for S in Ss:
                for vd in ([int(x) for x in args.vdepth.split(",")] if sc == "aica" else [0]):
                    run(sc, S, vd)
        else:
            run(sc, 0, 0)
    # summary: mean ms per scheme at its best S
    summ = {}
    for r in res["rows"]:
        key = r["scheme"] if "S" not in r else f"{r['scheme']}@S={r['S']}" + (
            f",vdepth={r['vdepth']}" if r["scheme"] == "aica" else "")
        summ.setdefault(key, []).append(r["ms"])
    res["mean_ms"] = {k: float(np.mean(v)) for k, v in summ.items()}
    pb = res["mean_ms"].get("pbox@S=0")
    if pb:
        res["speedup_vs_pbox"] = {k: pb / v for k, v in res["mean_ms"].items()}
    txt = json.dumps(res, indent=1)
    print(txt)
    if args.out:
        open(args.out, "w").write(txt)
    ctx.close()


if __name__ == "__main__":
    main()

"""Voxel-sharded single pivot on ONE GPU, rank by rank: for G = 1, 2, 4, 8, rank r's
model is the interleaved 256-voxel bricks b = r (mod G) (distributed.shard_voxels); each rank's map is the
single-pivot kernel's (am_compute) on its shard.  Reports per G the per-map device time of every rank
(median over the pivots, warm L2 and with L2 flushed before every call) -- the compute part of one
voxel-sharded step is the slowest rank's -- the ranks' live voxels, and checks that the OR of the G maps
is the whole model's map (the all_reduce(MAX) of distributed.run_sharded).  The collective itself (a
4 KB all_reduce over NVLink) needs G GPUs and is not measured here.
    python tools/shard_sweep.py C3 [C2 ...]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import scenes  # noqa: E402
import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402
from paper_conf_icpp_chenktkv19_b200.distributed import shard_voxels  # noqa: E402


def times(ctx, P, flush, s, out):
    warm, cold = [], []
    for mode, acc in (("warm", warm), ("cold", cold)):
        for rep in range(2):
            ev = []
            for i, p in enumerate(P):
                if mode == "cold":
                    with torch.cuda.stream(s):
                        flush.fill_((i + rep) & 255)
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(s)
                ctx.compute(p, out=out[i], stream=s)
                b.record(s)
                ev.append((a, b))
            s.synchronize()
            acc.extend(a.elapsed_time(b) * 1e3 for a, b in ev)
    return float(np.median(warm)), float(np.median(cold))


def main(names):
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    s = torch.cuda.Stream()
    for name in names:
        cfg = scenes.CONFIGS[name]
        C, H = cfg.leaves()
        P = cfg.pivots(16)
        whole = None
        for G in (1, 2, 4, 8):
            maps, rows = [], []
            for r in range(G):
                Cr, Hr = shard_voxels(C, H, r, G)
                ctx = am.Context(cfg.tool, cfg.m, cfg.n)
                ctx.upload(torch.from_numpy(np.ascontiguousarray(Cr)).cuda(), torch.from_numpy(np.ascontiguousarray(Hr)).cuda())
                out = torch.zeros((len(P), ctx.words), dtype=torch.int32, device="cuda")
                ctx.compute(P[0], out=out[0], stream=s)  # (first launch)
                w, c = times(ctx, P, flush, s, out)
                st = [ctx.compute(p, stats=True)[1] for p in P]
                maps.append(out.cpu().numpy().view(np.uint32).copy())
                rows.append((r, len(Hr), w, c, np.mean([x.voxels_live for x in st]), np.mean([x.voxels_streamed for x in st]),
                             np.mean([x.exact_tests for x in st])))
                ctx.close()
            comb = np.bitwise_or.reduce(np.stack(maps), axis=0)
            if G == 1:
                whole = comb
            same = bool(np.array_equal(comb, whole))
            wmax = max(x[2] for x in rows)
            cmax = max(x[3] for x in rows)
            print(f"{name} G={G}: per-map us, slowest rank: warm {wmax:.1f} flushed {cmax:.1f}; OR of the {G} maps "
                  f"{'==' if same else '!='} whole-model map", flush=True)
            for r, n, w, c, live, stream, ex in rows:
                print(f"   rank {r}: {n} voxels, warm {w:.1f} us, flushed {c:.1f} us, live {live:.0f}, streamed {stream:.0f},"
                      f" exact tests {ex:.0f}", flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or ["C3"])

"""Diagnostics: how many voxels survive the clear-map filter, per map quality.

Runs C3 (default) for a few pivots and prints, per configuration, the popcount
of the coarse-level map, the live count of the full stream and the stream time.
    python tools/probe_live.py [config] [npivots]
"""
import json
import os
import sys
import time

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402
import scenes  # noqa: E402
from paper_conf_icpp_chenktkv19_b200 import binding as B  # noqa: E402


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "C3"
    npiv = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    P = cfg.pivots(npiv)
    ctx = am.Context(cfg.tool, cfg.m, cfg.n)
    ctx.upload(torch.from_numpy(C).cuda(), torch.from_numpy(H).cuda())
    out = torch.zeros(ctx.words, dtype=torch.int32, device="cuda")
    res = []
    for T, ph in ((64, 2), (128, 2), (256, 2), (128, 1)):
        ctx.set_option(B.OPT_CMAP_T, T)
        ctx.set_option(B.OPT_PHASES, ph)
        for p in P:
            row = {"T": T, "levels": ph, "pivot": p.tolist()}
            ctx.set_option(B.OPT_DIAG, 1)
            w, _ = ctx.compute(p)
            row["coarse_bits"] = int(am.unpack(w, cfg.m, cfg.n).sum())
            ctx.set_option(B.OPT_DIAG, 0)
            for k in range(3):
                ctx.compute(p, out=out)
            ctx.set_option(B.OPT_KERNEL_TIMING, 1)
            ctx.kernel_time()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            for k in range(20):
                ctx.compute(p, out=out)
            torch.cuda.synchronize()
            row["am_ms"] = (time.perf_counter() - t0) / 20 * 1e3
            kms, kl = ctx.kernel_time()
            row["stream_ms"] = kms / max(kl, 1)
            ctx.set_option(B.OPT_KERNEL_TIMING, 0)
            w, st = ctx.compute(p, stats=True)
            row["final_bits"] = int(am.unpack(w, cfg.m, cfg.n).sum())
            row["live"] = st.voxels_live
            row["passed"] = st.voxels_streamed - st.voxels_skipped - st.voxels_culled
            row["rows"] = st.rows_rasterised
            row["band"] = st.band_pairs
            # lower bound: map from the final AM of the same pivot
            ctx.set_option(B.OPT_DIAG, 2)
            w2, st2 = ctx.compute(p, stats=True)
            assert np.array_equal(w2, w)
            row["live_finalmap"] = st2.voxels_live
            row["passed_finalmap"] = st2.voxels_streamed - st2.voxels_skipped - st2.voxels_culled
            ctx.set_option(B.OPT_KERNEL_TIMING, 1)
            ctx.kernel_time()
            for k in range(10):
                ctx.compute(p, out=out)
            kms, kl = ctx.kernel_time()
            row["stream_ms_finalmap"] = kms / max(kl, 1)
            ctx.set_option(B.OPT_KERNEL_TIMING, 0)
            ctx.set_option(B.OPT_DIAG, 0)
            print(json.dumps(row), flush=True)
            res.append(row)
    os.makedirs("gpurun_out", exist_ok=True)
    json.dump(res, open(f"gpurun_out/probe_{name}.json", "w"), indent=1)


if __name__ == "__main__":
    main()

"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck): single-pivot
maps (am_latency_kernel), a batch (the phase kernels + graph, with and without programmatic dependent
launches), the baseline, the stage-fused batch and the reuse path, the TMA-staged full-stream filters, on
one config.  python tools/sanitize_run.py C1|T_head [pivots]"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import scenes  # noqa: E402
import paper_conf_icpp_chenktkv19_b200 as am  # noqa: E402
from paper_conf_icpp_chenktkv19_b200 import binding as B  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C1"
npiv = int(sys.argv[2]) if len(sys.argv) > 2 else 4
cfg = scenes.CONFIGS[name]
C, H = cfg.leaves()
P = cfg.pivots(npiv)
ctx = am.Context(cfg.tool, cfg.m, cfg.n)
ctx.upload(C, H)
single = np.stack([ctx.compute(p, stats=True)[0] for p in P])
ctx.set_option(B.OPT_BATCH, npiv)
ctx.set_option(B.OPT_BATCH_LANES, 2)
assert np.array_equal(ctx.compute_batch(P), single)  # (defaults: level 0 fused, PDL, far-block bound)
assert np.array_equal(ctx.compute_batch(P), single)  # (graph replay)
ctx.set_option(B.OPT_PDL, 0)
assert np.array_equal(ctx.compute_batch(P), single)
ctx.set_option(B.OPT_PDL, 1)
ctx.set_option(B.OPT_STAGE_FUSION, 0)
assert np.array_equal(ctx.compute_batch(P), single)
ctx.set_option(B.OPT_STAGE_FUSION, 7)
ctx.set_option(B.OPT_REUSE, 1)
assert np.array_equal(ctx.compute_batch(P), single)
assert np.array_equal(ctx.compute_batch(P), single)
ctx.set_option(B.OPT_FUSED, 0)  # the stage-by-stage single-pivot path
assert np.array_equal(ctx.compute(P[0])[0], single[0])
ctx.set_option(B.OPT_BRICKS, 0)  # the full stream: LDG filter, then the TMA rings
for tma in (0, 1, 2, 3):
    ctx.set_option(B.OPT_STREAM_TMA, tma)
    assert np.array_equal(ctx.compute(P[0])[0], single[0]), tma
ctx.set_option(B.OPT_BRICKS, 1)
ctx.compute_baseline(P[0])
ctx.close()
print(f"sanitize_run {name}: {npiv} pivots, single / batched (PDL on, off; level 0 fused, split) / stage-fused + "
      f"reuse / stage path / full stream LDG + 3 TMA rings / baseline ok")

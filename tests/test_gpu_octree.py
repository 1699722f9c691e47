"""GPU parity of the paper's own orientation-per-thread schemes (SURVEY.md 8(f)
NEXT 3; Alg. 2): PBox, optimized PBox, PICA, MICA
and AICA over the octree built from the leaves.  Every scheme falls back to the
exact test, so each must match the fp64 oracle on every robust cell (zero
mismatches), exactly like am_compute.
"""
import numpy as np
import pytest

import oracle
import scenes

pytestmark = pytest.mark.gpu

SCHEMES = ["pbox", "pbox_aabb", "pica", "mica", "aica"]


@pytest.fixture(scope="module")
def am(gpu):
    import paper_conf_icpp_chenktkv19_b200 as am
    return am


def _ctx(am, cfg, C, H):
    ctx = am.Context(cfg.tool, cfg.m, cfg.n, device=0)
    ctx.upload(C, H)
    return ctx


@pytest.mark.parametrize("name,npiv", [("C1", 2), ("T_head", 2), ("T_head4", 1), ("T_imp", 1)])
def test_schemes_match_oracle(am, name, npiv):
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    nn = ctx.build_octree(cfg.lo, cfg.size)
    assert nn > len(H)  # leaves + interior nodes
    for p in cfg.pivots(npiv):
        S = oracle.am_states(C, H, cfg.tool, p, cfg.m, cfg.n)
        robust = S != 1
        ref = ctx.am(p)
        for sc in SCHEMES:
            for Sl, vd in ((0, 0), (4, 0), (64, 2)):
                if sc not in ("mica", "aica") and (Sl, vd) != (0, 0):
                    continue
                w, st = ctx.compute_octree(p, sc, S=Sl, vdepth=vd, stats=True)
                g = am.unpack(w, cfg.m, cfg.n)
                mism = int(((g == 1) != (S == 2))[robust].sum())
                assert mism == 0, (name, sc, Sl, vd, mism)
                # same map as the streaming path outside the band
                assert int((g != ref)[robust].sum()) == 0
                assert st["nodes_popped"] >= cfg.m * cfg.n and st["max_popped_per_thread"] >= 1
                if sc in ("pbox", "pbox_aabb"):
                    assert st["ica_evals"] == 0
                if sc == "pbox":
                    assert st["box_tests"] == st["nodes_popped"]
                if sc == "mica" and Sl == 64:
                    assert st["ica_evals"] == 0  # every node memoised
    ctx.close()


def test_scheme_work_ordering(am):
    """The paper's ordering of work (Table 3, Fig. 13): the ICA schemes call
    CHECKBOX far less than PBox; the AABB reject removes box tests."""
    cfg = scenes.CONFIGS["T_head"]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    ctx.build_octree(cfg.lo, cfg.size)
    p = cfg.pivots(1)[0]
    st = {sc: ctx.compute_octree(p, sc, S=4, vdepth=1, stats=True)[1] for sc in SCHEMES}
    assert st["pbox_aabb"]["box_tests"] < st["pbox"]["box_tests"]
    assert st["pica"]["box_tests"] * 3 < st["pbox"]["box_tests"]  # 4.7x at 1.25 mm cells
    assert st["mica"]["box_tests"] == st["pica"]["box_tests"]
    assert st["mica"]["ica_evals"] < st["pica"]["ica_evals"]
    ctx.close()


def test_octree_build_rejects_non_octree_input(am):
    cfg = scenes.CONFIGS["C1"]
    C, H = cfg.leaves()
    ctx = _ctx(am, cfg, C, H)
    with pytest.raises(am.AMError):
        ctx.build_octree(cfg.lo, cfg.size * 1.37)  # sizes are not root / 2^(l+1)
    with pytest.raises(am.AMError):
        ctx.build_octree((cfg.lo[0] + 0.3, cfg.lo[1], cfg.lo[2]), cfg.size)  # centres off the cells
    with pytest.raises(am.AMError):
        ctx.compute_octree(cfg.pivots(1)[0], "pbox")  # no octree after the failed builds
    # overlapping leaves: a cell and one of its children
    C2 = np.concatenate([C, C[:1] + H[:1, None] * 0.5]).astype(np.float32)
    H2 = np.concatenate([H, H[:1] * 0.5]).astype(np.float32)
    ctx.upload(C2, H2)
    with pytest.raises(am.AMError):
        ctx.build_octree(cfg.lo, cfg.size)
    ctx.close()


def test_empty_and_enclosed(am):
    cfg = scenes.CONFIGS["C1"]
    ctx = am.Context(cfg.tool, 16, 16, device=0)
    ctx.upload(np.zeros((0, 3), np.float32), np.zeros(0, np.float32))
    assert ctx.build_octree(cfg.lo, cfg.size) == 0
    w, _ = ctx.compute_octree((0.0, 0.0, 0.0), "aica", S=3)
    assert not w.any()
    # the pivot inside a leaf: every orientation collides, in every scheme
    ctx.upload(np.array([[0.5, 0.5, 0.5]], np.float32), np.array([0.5], np.float32))
    ctx.build_octree((-32.0, -32.0, -32.0), 64.0)
    for sc in SCHEMES:
        w, _ = ctx.compute_octree((0.6, 0.4, 0.5), sc, S=2)
        assert am.unpack(w, 16, 16).all(), sc
    ctx.close()

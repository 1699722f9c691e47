"""Input-generator invariants (scenes/ holds no method arithmetic)."""
import numpy as np

import scenes


def test_c1_leaf_count_and_sizes():
    C, H = scenes.CONFIGS["C1"].leaves()
    assert len(H) == 27208
    assert H.min() == 0.5 and C.dtype == np.float32


def test_leaves_cover_the_surface_and_are_disjoint():
    C, H = scenes.octree_leaves("head", (), (-40, -40, -40), 80.0, 5)
    lo = C - H[:, None]
    hi = C + H[:, None]
    # disjoint: total volume equals the volume of the union on a fine sample grid
    g = np.linspace(-39.9, 39.9, 41)
    X, Y, Z = np.meshgrid(g, g, g, indexing="ij")
    P = np.stack([X.ravel(), Y.ravel(), Z.ravel()], 1)
    f = scenes.sdf("head", P)
    inside = P[f < 0]
    cnt = np.zeros(len(inside), int)
    for a, b in zip(lo, hi):
        cnt += np.all((inside >= a) & (inside <= b), axis=1)
    assert (cnt >= 1).all()  # every interior sample point is covered


def test_morton_order_is_depth_first():
    C, H = scenes.octree_leaves("sphere", (10.0,), (-16, -16, -16), 32.0, 4)

    def key(c, lo=-16.0, cell=2.0, bits=4):
        q = ((c - lo) / cell).astype(np.int64)
        k = np.zeros(len(c), np.int64)
        for b in range(bits):
            for a in range(3):
                k |= ((q[:, a] >> b) & 1) << (3 * b + a)
        return k
    # keys of each leaf's lowest-corner finest cell are non-decreasing
    corner = C - H[:, None] + 1.0
    k = key(corner)
    assert np.all(np.diff(k) > 0)


def test_pivots_are_on_the_offset_path_and_outside_the_voxels():
    cfg = scenes.CONFIGS["T_head"]
    C, H = cfg.leaves()
    P = cfg.pivots(6)
    f = scenes.sdf(cfg.model, P.astype(np.float64))
    off = max(cfg.offset, 2 * np.sqrt(3) * cfg.min_half() + 0.05)
    assert (f >= off).all() and (f < off + 0.01).all()
    for p in P:
        inside = np.all(np.abs(C - p[None, :]) <= H[:, None], axis=1)
        assert not inside.any()
    # seeded: same seeds -> same pivots
    assert np.array_equal(P, cfg.pivots(6))


def test_pivots_at_matches_pivots_and_toolpath_is_continuous():
    """pivots_at(indices) gives pivots(n)[indices] (a rank generates only its own); the toolpath's
    pivots are on the offset surface, outside every voxel, and consecutive ones are neighbours."""
    cfg = scenes.CONFIGS["T_head"]
    P = cfg.pivots(7)
    assert np.array_equal(cfg.pivots_at(range(7)), P)
    assert np.array_equal(cfg.pivots_at([5, 2]), P[[5, 2]])
    C, H = cfg.leaves()
    T = cfg.toolpath(1024)
    off = max(cfg.offset, 2 * np.sqrt(3) * cfg.min_half() + 0.05)
    f = scenes.sdf(cfg.model, T.astype(np.float64))
    assert (f >= off).all()
    for p in T[::64]:
        assert not np.all(np.abs(C - p[None, :]) <= H[:, None], axis=1).any()
    step = np.linalg.norm(np.diff(T, axis=0), axis=1)
    rnd = np.linalg.norm(P[:, None, :] - P[None, :, :], axis=2)[np.triu_indices(7, 1)]
    assert np.median(step) < 0.1 * np.median(rnd)  # neighbours, unlike the seeded pivots (~40 mm apart)

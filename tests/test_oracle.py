"""Pins for the fp64 oracle (CPU only).

Every check here compares the oracle with something other than itself: closed
forms derived from the geometry (tests/golden/closed_forms.json), an
independent convex-QP solver (scipy SLSQP), dense point sampling, the analytic
sphere cap, symmetry, special cases and metamorphic invariances
(DESIGN.md "Oracle pins").
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
import scenes

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "closed_forms.json")))


def _rot_dir(theta, gamma):
    return np.array([math.sin(theta) * math.cos(gamma), math.sin(theta) * math.sin(gamma), math.cos(theta)])


# ---------------------------------------------------------------- P1 closed forms

@pytest.mark.parametrize("gamma_key,gammas", [
    ("theta_star_gamma0", [0.0, 0.5 * math.pi, math.pi, 1.5 * math.pi]),
    ("theta_star_gamma45", [0.25 * math.pi, 0.75 * math.pi, 1.25 * math.pi, 1.75 * math.pi]),
])
def test_on_axis_closed_form(gamma_key, gammas):
    g = GOLD["on_axis"]
    D, h, R = g["D"], g["h"], g["R"]
    th = g[gamma_key]
    # recompute the golden value from its derivation (guards the fixture itself)
    w = h if gamma_key.endswith("0") else math.sqrt(2) * h
    assert th == pytest.approx(math.atan2(w, D - h) + math.asin(R / math.hypot(D - h, w)), abs=1e-12)
    v = np.array([0.0, 0.0, D])
    for gam in gammas:
        for dth, expect in ((-2e-9, True), (+2e-9, False)):
            d = _rot_dir(th + dth, gam)
            assert oracle.box_cyl_hit(v, h, d, 0.0, 500.0, R) is expect, (gam, dth)
        # the axis distance at the critical angle is R
        assert oracle.axis_dist(v, h, _rot_dir(th, gam), 0.0, 500.0) == pytest.approx(R, abs=1e-9)


def test_on_axis_sandwich():
    g = GOLD["on_axis"]
    assert g["sandwich_inscribed"] < g["theta_star_gamma0"] < g["theta_star_gamma45"] < g["sandwich_circumscribed"]


def test_cap_and_side_contact():
    R, L, h = 6.35, 100.0, 0.5
    z = np.array([0.0, 0.0, 1.0])
    for t in (1e-7, 1e-4, 0.3):
        # box beyond the tool end along the axis
        assert oracle.box_cyl_hit([0, 0, L + h - t], h, z, 0.0, L, R)
        assert not oracle.box_cyl_hit([0, 0, L + h + t], h, z, 0.0, L, R)
        # box beside the cylinder
        assert oracle.box_cyl_hit([R + h - t, 0, 50.0], h, z, 0.0, L, R)
        assert not oracle.box_cyl_hit([R + h + t, 0, 50.0], h, z, 0.0, L, R)
        # box behind the pivot (the tip's end face is at axial 0)
        assert oracle.box_cyl_hit([0, 0, -h + t], h, z, 0.0, L, R)
        assert not oracle.box_cyl_hit([0, 0, -h - t], h, z, 0.0, L, R)
        # box diagonal to the rim: corner (x, x, z) touches the rim circle at 45 deg
        c = R / math.sqrt(2)
        assert oracle.box_cyl_hit([c + h - t, c + h - t, 50.0], h, z, 0.0, L, R)
        assert not oracle.box_cyl_hit([c + h + t, c + h + t, 50.0], h, z, 0.0, L, R)
    # touching exactly counts as a collision (closed sets, reading G7)
    assert oracle.box_cyl_hit([R + h, 0, 50.0], h, z, 0.0, L, R)


# ---------------------------------------------------------------- independent QP

def _qp_dist(v, h, d, z0, z1):
    from scipy.optimize import minimize
    d = np.asarray(d, float)
    P = np.eye(3) - np.outer(d, d)

    def f(x):
        y = P @ x
        return float(y @ y)

    def g(x):
        return 2.0 * (P @ x)
    bounds = [(v[k] - h, v[k] + h) for k in range(3)]
    cons = [{"type": "ineq", "fun": lambda x: x @ d - z0, "jac": lambda x: d},
            {"type": "ineq", "fun": lambda x: z1 - x @ d, "jac": lambda x: -d}]
    best = math.inf
    rng = np.random.default_rng(0)
    for s in range(6):
        x0 = np.asarray(v, float) + rng.uniform(-h, h, 3)
        r = minimize(f, x0, jac=g, bounds=bounds, constraints=cons, method="SLSQP",
                     options={"ftol": 1e-16, "maxiter": 500})
        x = np.clip(r.x, [b[0] for b in bounds], [b[1] for b in bounds])
        if z0 - 1e-9 <= x @ d <= z1 + 1e-9:
            best = min(best, math.sqrt(max(f(x), 0.0)))
    return best


def test_axis_dist_vs_convex_qp():
    rng = np.random.default_rng(1234)
    checked = 0
    for _ in range(120):
        d = rng.normal(size=3)
        d /= np.linalg.norm(d)
        v = rng.uniform(-6, 6, 3)
        h = rng.uniform(0.2, 2.0)
        z0 = rng.uniform(-5, 3)
        z1 = z0 + rng.uniform(0.1, 6)
        dist = oracle.axis_dist(v, h, d, z0, z1)
        # emptiness from the support function of the cube (independent)
        s = h * np.abs(d).sum()
        empty = (v @ d + s < z0) or (v @ d - s > z1)
        assert (dist < 0) == empty
        if empty:
            continue
        q = _qp_dist(v, h, d, z0, z1)
        assert dist == pytest.approx(q, abs=2e-6), (v, h, d, z0, z1)
        checked += 1
    assert checked > 40


def test_axis_dist_lower_bounds_sampled_points():
    """Every sampled point of box cap slab is at least `dist` from the axis (oracle = min)."""
    rng = np.random.default_rng(7)
    for _ in range(200):
        d = rng.normal(size=3)
        d /= np.linalg.norm(d)
        v = rng.uniform(-4, 4, 3)
        h = rng.uniform(0.2, 1.5)
        z0 = rng.uniform(-4, 2)
        z1 = z0 + rng.uniform(0.1, 5)
        dist = oracle.axis_dist(v, h, d, z0, z1)
        pts = v + rng.uniform(-h, h, (4000, 3))
        # include the cube's vertices
        corners = v + h * np.array([[sx, sy, sz] for sx in (-1, 1) for sy in (-1, 1) for sz in (-1, 1)])
        pts = np.concatenate([pts, corners])
        a = pts @ d
        inslab = (a >= z0) & (a <= z1)
        if not inslab.any():
            continue
        assert dist >= 0
        rho = np.linalg.norm(pts[inslab] - a[inslab, None] * d[None, :], axis=1)
        assert rho.min() >= dist - 1e-12
        # and the sampled minimum is not far above it (dense sampling)
        assert rho.min() <= dist + 0.6 * h * 2


# ---------------------------------------------------------------- 3-state margin

def test_robust_states_survive_rotation_within_delta():
    rng = np.random.default_rng(99)
    tool = scenes.TOOL_3CYL
    delta = oracle.DELTA
    zs = np.cumsum([0.0] + [t[1] for t in tool])
    n_robust = 0
    for _ in range(400):
        # near-contact pairs: voxel near the side of a random cylinder
        k = rng.integers(0, len(tool))
        R, H = tool[k]
        ax = rng.uniform(zs[k], zs[k + 1])
        h = rng.uniform(0.01, 0.5)
        gap = rng.normal() * 2e-4 * ax
        v_loc = np.array([R + h + gap, 0.0, ax])
        d = _rot_dir(rng.uniform(0.1, 3.0), rng.uniform(0, 2 * math.pi))
        # place the voxel in the frame of d
        e1 = np.cross(d, [0.3, 0.4, 0.5]); e1 /= np.linalg.norm(e1)
        e2 = np.cross(d, e1)
        v = v_loc[0] * e1 + v_loc[1] * e2 + v_loc[2] * d
        st = oracle.pair_state(v, h, d, tool, delta)
        if st == 1:
            continue
        n_robust += 1
        for _ in range(6):
            # rotate d by an angle < delta about a random axis
            a = rng.normal(size=3)
            a -= (a @ d) * d
            a /= np.linalg.norm(a)
            ang = delta * rng.uniform(0.0, 0.999)
            d2 = math.cos(ang) * d + math.sin(ang) * a
            hit = any(oracle.box_cyl_hit(v, h, d2, zs[q], zs[q + 1], tool[q][0]) for q in range(len(tool)))
            assert hit == (st == 2)
    assert n_robust > 100


def test_margin_covers_far_contact_points():
    """A big box whose contact face extends to axial 25 mm: a rotation by delta
    about the pivot sweeps the tool side by up to 25 * delta, beyond |c - p| * delta,
    so the margin must use |c - p| + sqrt(3) h (reading G10)."""
    R, h, zc, gap = 6.35, 5.0, 20.0, 2.45e-4
    v = np.array([R + h + gap, 0.0, zc])
    z = np.array([0.0, 0.0, 1.0])
    tool = ((R, 150.0),)
    ang = 0.999 * oracle.DELTA
    d2 = np.array([math.sin(ang), 0.0, math.cos(ang)])  # tilt toward the box
    assert not oracle.box_cyl_hit(v, h, z, 0.0, 150.0, R)
    assert oracle.box_cyl_hit(v, h, d2, 0.0, 150.0, R)
    assert oracle.pair_state(v, h, z, tool) == 1  # band, not robust-miss


def test_shortcuts_are_exact():
    c = scenes.CONFIGS["T_head"]
    C, H = c.leaves()
    piv = c.pivots(2)
    for p in piv:
        a = oracle.am_states(C, H, c.tool, p, 24, 28, shortcuts=True)
        b = oracle.am_states(C, H, c.tool, p, 24, 28, shortcuts=False)
        assert np.array_equal(a, b)


def _nearest_first(C, H, p):
    """The voxels in order of D - sqrt(3) h from the pivot (the AM is a plain OR over voxels, so
    the order is free -- test_permutation_invariance; blocked cells then stop at a near voxel)."""
    o = np.argsort(np.linalg.norm(C.astype(np.float64) - np.asarray(p, np.float64)[None, :], axis=1)
                   - math.sqrt(3.0) * H, kind="stable")
    return np.ascontiguousarray(C[o]), np.ascontiguousarray(H[o])


@pytest.mark.parametrize("name", ["C1", "C2"])
def test_shortcuts_are_exact_on_configs(name):
    """the exact-safe sphere shortcuts agree bit for bit with the plain
    clip-project-hull path on C1 and C2 -- every cell of the full map of two pivots each (C2:
    1.95M voxels), the cell states (0 / 1 / 2) compared exactly."""
    cfg = scenes.CONFIGS[name]
    C, H = cfg.leaves()
    for p in cfg.pivots(2):
        Cs, Hs = _nearest_first(C, H, p)
        a = oracle.am_states(Cs, Hs, cfg.tool, p, cfg.m, cfg.n, shortcuts=True)
        b = oracle.am_states(Cs, Hs, cfg.tool, p, cfg.m, cfg.n, shortcuts=False)
        assert np.array_equal(a, b), (name, p, int((a != b).sum()))
        assert (a == 0).any() and (a == 2).any()  # both decisions exercised


def test_shortcuts_are_exact_pairs_near_the_cones():
    """Pair-level identity of the shortcuts (stronger than per cell: no hit can hide behind
    another voxel's) on C2 voxels near the pivot, with directions spread over and around each
    voxel's blocked cone (angles up to 1.3 x asin((R_max + sqrt3 h) / D)), paper 4-cyl tool."""
    cfg = scenes.CONFIGS["C2"]
    C, H = cfg.leaves()
    rng = np.random.default_rng(5)
    tool = scenes.TOOL_PAPER4
    Rmax = max(r for r, _ in tool)
    states = np.zeros(3, int)
    for p in cfg.pivots(2):
        Cs, Hs = _nearest_first(C, H, p)
        pick = np.concatenate([np.arange(400), rng.choice(len(Hs), 400, replace=False)])
        for q in pick:
            v = Cs[q].astype(np.float64) - p.astype(np.float64)
            D = np.linalg.norm(v)
            u = v / D
            a = np.array([1.0, 0.0, 0.0]) if abs(u[0]) < 0.9 else np.array([0.0, 1.0, 0.0])
            e1 = np.cross(u, a)
            e1 /= np.linalg.norm(e1)
            e2 = np.cross(u, e1)
            top = 1.3 * math.asin(min(1.0, (Rmax + math.sqrt(3.0) * Hs[q]) / D))
            for th, az in zip(rng.uniform(0.0, min(top, math.pi), 12), rng.uniform(0, 2 * math.pi, 12)):
                d = math.cos(th) * u + math.sin(th) * (math.cos(az) * e1 + math.sin(az) * e2)
                s1 = oracle.pair_state(v, Hs[q], d, tool, shortcuts=True)
                s0 = oracle.pair_state(v, Hs[q], d, tool, shortcuts=False)
                assert s1 == s0, (q, th, az, s1, s0)
                states[s1] += 1
    assert states[0] > 1000 and states[2] > 1000, states  # (band pairs are a 1e-5 rad sliver)


# ---------------------------------------------------------------- P3 sphere cap

def _theta_c(Rs, Dp, R):
    if math.sqrt(Dp * Dp - Rs * Rs) <= R:
        return math.acos(Rs / Dp)
    return math.asin((Dp * Dp + R * R - Rs * Rs) / (2 * Dp * R))


def test_sphere_cap_C1():
    g = GOLD["sphere_cap_C1"]
    c = scenes.CONFIGS["C1"]
    C, H = c.leaves()
    assert len(H) == 27208  # SURVEY 8(d) C1 leaf count
    Rs, h, Dp, R = g["Rs"], g["h"], g["Dp"], g["R"]
    lo = _theta_c(Rs + 2 * math.sqrt(3) * h, Dp, R)
    hi = _theta_c(Rs, Dp, R)
    assert math.degrees(lo) == pytest.approx(g["theta_lo_deg"], abs=1e-9)
    assert math.degrees(hi) == pytest.approx(g["theta_hi_deg"], abs=1e-9)
    # the voxel model is sandwiched between the two balls
    rad = np.linalg.norm(C.astype(np.float64), axis=1)
    assert (rad + math.sqrt(3) * H <= Rs + 2 * math.sqrt(3) * h + 1e-9).all()
    S = oracle.am_states(C, H, c.tool, (0, 0, Dp), c.m, c.n)
    phi = (np.arange(c.m) + 0.5) * math.pi / c.m
    assert (S[phi < lo - 1e-4] == 0).all()
    assert (S[phi > hi + 1e-4] == 2).all()
    assert (phi < lo - 1e-4).sum() >= 3 and (phi > hi + 1e-4).sum() >= 26


# ---------------------------------------------------------------- direction conventions

@pytest.mark.parametrize("phi0,gam0", [(1.0, 0.7), (2.2, 4.0), (0.6, 2.5)])
def test_single_voxel_sandwich_and_conventions(phi0, gam0):
    """A lone voxel at direction (phi0, gamma0): the blocked cells form a cap
    centred there, between the inscribed- and circumscribed-sphere cones
    (Alg. 1, Fig. 8).  Pins phi-from-+z, gamma-from-+x
    toward +y, row = phi index, col = gamma index."""
    D, h, R = 40.0, 0.9, 6.35
    tool = ((R, 150.0),)
    m, n = 48, 64
    v = D * _rot_dir(phi0, gam0)
    piv = np.array([1.5, -2.0, 0.75], dtype=np.float32)
    cen = (v + piv).astype(np.float32)[None, :]
    S = oracle.am_states(cen, np.array([h], np.float32), tool, piv, m, n)
    vd = (cen[0].astype(np.float64) - piv)
    vd /= np.linalg.norm(vd)
    Dd = np.linalg.norm(cen[0].astype(np.float64) - piv)
    t_in = math.asin((R + h) / Dd)
    t_out = math.asin((R + math.sqrt(3) * h) / Dd)
    n_in = n_out = 0
    for i in range(m):
        for j in range(n):
            th = math.acos(np.clip(oracle.cell_dir(i, j, m, n) @ vd, -1, 1))
            if th < t_in - 1e-4:
                assert S[i, j] == 2
                n_in += 1
            elif th > t_out + 1e-4:
                assert S[i, j] == 0
                n_out += 1
    assert n_in >= 3 and n_out > m * n // 2
    # the cell holding the voxel direction is blocked
    i0 = int(phi0 / (math.pi / m))
    j0 = int(gam0 / (2 * math.pi / n))
    assert S[i0, j0] == 2


def test_cell_dir_convention():
    m, n = 8, 12
    d = oracle.cell_dir(0, 0, m, n)
    phi, gam = 0.5 * math.pi / m, 0.5 * 2 * math.pi / n
    assert np.allclose(d, [math.sin(phi) * math.cos(gam), math.sin(phi) * math.sin(gam), math.cos(phi)])


# ---------------------------------------------------------------- P4 symmetry

def test_symmetry_C1_offaxis_scene():
    c = scenes.CONFIGS["C1"]
    C, H = c.leaves()
    S = oracle.am_states(C, H, c.tool, (0, 0, 30.0), c.m, 64)
    n = 64
    j = np.arange(n)
    for perm in ((j + n // 4) % n, (n // 2 - 1 - j) % n, (n - 1 - j) % n):
        A, B = S, S[:, perm]
        robust = (A != 1) & (B != 1)
        assert np.array_equal(A[robust], B[robust])


# ---------------------------------------------------------------- P5 special cases

def test_empty_and_out_of_reach():
    tool = scenes.TOOL_3CYL
    S = oracle.am_states(np.zeros((0, 3), np.float32), np.zeros(0, np.float32), tool, (0, 0, 0), 16, 16)
    assert (S == 0).all()
    far = np.array([[400.0, 0, 0], [0, -300.0, 100.0]], np.float32)
    S = oracle.am_states(far, np.array([1.0, 2.0], np.float32), tool, (0, 0, 0), 16, 16)
    assert (S == 0).all()


def test_pivot_inside_voxel_blocks_everything():
    S = oracle.am_states(np.array([[0.3, -0.2, 0.1]], np.float32), np.array([0.5], np.float32),
                         scenes.TOOL_3CYL, (0, 0, 0), 16, 20)
    assert (S == 2).all()


def test_enclosing_shell_blocks_everything():
    C, H = scenes.octree_leaves("shell", (24.0, 20.0), (-32, -32, -32), 64.0, 5)
    assert len(H) > 0
    S = oracle.am_states(C, H, scenes.TOOL_3CYL, (0.5, -0.25, 0.3), 16, 16)
    assert (S == 2).all()


# ---------------------------------------------------------------- P6 metamorphic

def _robust_equal(A, B):
    robust = (A != 1) & (B != 1)
    return np.array_equal(A[robust], B[robust])


def test_permutation_invariance():
    c = scenes.CONFIGS["T_head"]
    C, H = c.leaves()
    p = c.pivots(1)[0]
    perm = np.random.default_rng(5).permutation(len(H))
    A = oracle.am_states(C, H, c.tool, p, 32, 32)
    B = oracle.am_states(C[perm], H[perm], c.tool, p, 32, 32)
    assert np.array_equal(A, B)


def test_split_into_children_invariance():
    c = scenes.CONFIGS["T_head"]
    C, H = c.leaves()
    p = c.pivots(3)[2]
    big = H > H.min()
    kids_c, kids_h = [], []
    for s in range(8):
        off = np.stack([np.where(s & 1, 1, -1), np.where(s & 2, 1, -1), np.where(s & 4, 1, -1)]).astype(np.float32)
        kids_c.append(C[big] + 0.5 * H[big, None] * off[None, :])
        kids_h.append(0.5 * H[big])
    C2 = np.concatenate([C[~big]] + kids_c)
    H2 = np.concatenate([H[~big]] + kids_h)
    A = oracle.am_states(C, H, c.tool, p, 32, 32)
    B = oracle.am_states(C2, H2, c.tool, p, 32, 32)
    # the parent's robust states are preserved by the children
    robustA = A != 1
    assert np.array_equal(A[robustA], B[robustA])


def test_interior_leaf_removal_invariance():
    c = scenes.CONFIGS["T_head"]
    C, H = c.leaves()
    f = scenes.sdf("head", C.astype(np.float64))
    interior = f < -np.sqrt(3) * H
    assert interior.sum() > 100
    for p in c.pivots(3):
        A = oracle.am_states(C, H, c.tool, p, 32, 32)
        B = oracle.am_states(C[~interior], H[~interior], c.tool, p, 32, 32)
        assert _robust_equal(A, B)


def test_monotone_in_voxels_and_radius():
    c = scenes.CONFIGS["T_head"]
    C, H = c.leaves()
    p = c.pivots(1)[0]
    half = np.arange(len(H)) % 2 == 0
    A = oracle.am_states(C[half], H[half], c.tool, p, 32, 32)
    B = oracle.am_states(C, H, c.tool, p, 32, 32)
    assert not ((A == 2) & (B == 0)).any()
    fat = tuple((r + 1.0, hh) for r, hh in c.tool)
    F = oracle.am_states(C, H, fat, p, 32, 32)
    assert not ((B == 2) & (F == 0)).any()


def test_pack_unpack_layout():
    rng = np.random.default_rng(3)
    for m, n in ((3, 1), (5, 32), (4, 33), (7, 100)):
        a = (rng.random((m, n)) < 0.5).astype(np.uint8)
        w = oracle.pack_bits(a)
        assert w.shape == (m, (n + 31) // 32)
        # bit j of row i is bit (j & 31) of word i*W + j>>5 (reading G2)
        i, j = m - 1, n - 1
        assert (int(w[i, j >> 5]) >> (j & 31)) & 1 == a[i, j]
        assert np.array_equal(oracle.unpack_bits(w.reshape(-1), m, n), a)

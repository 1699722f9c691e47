"""Seeded synthetic inputs for the AM hot path (shared by tests, bench and smoke).

This module is INPUT GENERATION ONLY.  It holds none of the method's arithmetic
(no cones, no cylinder-box tests): analytic signed-distance models, the adaptive
octree leaf rule (``octree.c``), tool definitions and the 1 mm pivot path.  Both
the CUDA path's tests and the oracle's tests draw their inputs from here, and
neither side's code lives here.

Recipe:

* models are Lipschitz-1 distance bounds shaped like the paper's CAD benchmarks
  (Table 1): a sphere (C1), a head (C2/C3), a turbine-blade-like
  thin wall (C4) and an impeller (C5);
* leaves: cells with |f(c)| <= sqrt(3) h are split down to max depth, cells with
  f < -sqrt(3) h are full interior leaves, the rest is dropped; Morton order;
* tools: PAPER.md L311 lists radii (31.5, 20, 6.225, 6.35) and heights
  (22.1, 78, 76.2, 25.4) holder->tip; from the pivot outward (reading G3) the
  3-cylinder tool is tip/shank/holder;
* pivots: "each point on the path having a 1 mm distance from the surface"
  (L311): a seeded direction u is marched from the model centre to the first
  point whose distance bound reaches the offset (model seed 0, pivot seed 1+k).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass, field

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libscenes.so")
_lib = None

MODELS = {"sphere": 0, "head": 1, "blade": 2, "impeller": 3, "shell": 4}

# (radius, height) from the pivot outward -- PAPER.md L311, reading G3
TOOL_1CYL = ((6.35, 150.0),)
TOOL_3CYL = ((6.35, 25.4), (6.225, 76.2), (20.0, 78.0))
TOOL_PAPER4 = TOOL_3CYL + ((31.5, 22.1),)


def build(force: bool = False) -> str:
    """Compile octree.c into libscenes.so (plain gcc + OpenMP)."""
    src = os.path.join(_HERE, "octree.c")
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", src, "-o", _LIB_PATH, "-lm"])
    return _LIB_PATH


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB_PATH)
        lib.scene_octree.restype = ctypes.c_int
        lib.scene_octree.argtypes = [
            ctypes.c_int, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_double),
            ctypes.c_double, ctypes.c_int, ctypes.POINTER(ctypes.POINTER(ctypes.c_float)),
            ctypes.POINTER(ctypes.POINTER(ctypes.c_float)), ctypes.POINTER(ctypes.c_int64)]
        lib.scene_sdf.restype = None
        lib.scene_sdf.argtypes = [ctypes.c_int, ctypes.POINTER(ctypes.c_double),
                                  ctypes.POINTER(ctypes.c_double), ctypes.c_int64,
                                  ctypes.POINTER(ctypes.c_double)]
        lib.scene_free.argtypes = [ctypes.c_void_p]
        _lib = lib
    return _lib


def _dptr(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def _params(p):
    a = np.zeros(8, dtype=np.float64)
    a[: len(p)] = p
    return a


def octree_leaves(model: str, params=(), lo=(-1.0, -1.0, -1.0), size=2.0, depth=4):
    """Leaves (centres float32[N,3], half sizes float32[N]) of the model's adaptive octree."""
    lib = _load()
    pa = _params(params)
    lo_a = np.asarray(lo, dtype=np.float64)
    pc = ctypes.POINTER(ctypes.c_float)()
    ph = ctypes.POINTER(ctypes.c_float)()
    n = ctypes.c_int64(0)
    rc = lib.scene_octree(MODELS[model], _dptr(pa), _dptr(lo_a), float(size), int(depth),
                          ctypes.byref(pc), ctypes.byref(ph), ctypes.byref(n))
    if rc != 0:
        raise MemoryError("scene_octree failed")
    N = n.value
    try:
        c = np.ctypeslib.as_array(pc, shape=(max(N, 1) * 3,))[: N * 3].copy().reshape(N, 3)
        h = np.ctypeslib.as_array(ph, shape=(max(N, 1),))[:N].copy()
    finally:
        lib.scene_free(ctypes.cast(pc, ctypes.c_void_p))
        lib.scene_free(ctypes.cast(ph, ctypes.c_void_p))
    return c, h


def sdf(model: str, points, params=()) -> np.ndarray:
    """Distance bound f at points (float64[...,3]); f > 0 outside."""
    lib = _load()
    pts = np.ascontiguousarray(np.asarray(points, dtype=np.float64).reshape(-1, 3))
    out = np.empty(len(pts), dtype=np.float64)
    pa = _params(params)
    lib.scene_sdf(MODELS[model], _dptr(pa), _dptr(pts), len(pts), _dptr(out))
    return out.reshape(np.asarray(points).shape[:-1])


def _march_to_offset(model, params, u, offset, c):
    """The first point along c + t u (0.25 mm steps, then bisection) whose distance bound reaches
    `offset` and stays there for 2 mm (skips blade gaps); f(pivot) >= offset."""
    ts = np.arange(0.0, 400.0, 0.25)
    f = sdf(model, c[None, :] + ts[:, None] * u[None, :], params)
    idx = np.nonzero(f >= offset)[0]
    j = None
    for i in idx:
        if i > 0 and np.all(f[i: i + 8] >= offset):
            j = i
            break
    if j is None:
        j = idx[-1]
    a, b = ts[j - 1], ts[j]
    for _ in range(50):
        mid = 0.5 * (a + b)
        if sdf(model, (c + mid * u)[None, :], params)[0] >= offset:
            b = mid
        else:
            a = mid
    p = (c + b * u).astype(np.float32)
    # float32 rounding must not bring the pivot closer than the offset
    while sdf(model, p.astype(np.float64)[None, :], params)[0] < offset:
        b += 1e-4
        p = (c + b * u).astype(np.float32)
    return p


def path_pivots(model: str, params, count: int, offset: float, seed0: int = 1,
                centre=(0.0, 0.0, 0.0)):
    """Pivots on the offset path: pivot k uses seed seed0 + k.

    A seeded direction u is marched from ``centre`` in 0.25 mm steps until the
    distance bound reaches ``offset``; the crossing is refined by bisection and
    the pivot is taken on the outside end, so f(pivot) >= offset.
    """
    out = np.empty((count, 3), dtype=np.float32)
    c = np.asarray(centre, dtype=np.float64)
    for k in range(count):
        rng = np.random.default_rng(seed0 + k)
        u = rng.normal(size=3)
        u /= np.linalg.norm(u)
        out[k] = _march_to_offset(model, params, u, offset, c)
    return out


def toolpath_pivots(model: str, params, count: int, offset: float, centre=(0.0, 0.0, 0.0), turns: float = 16.0):
    """A continuous toolpath on the offset surface (PAPER.md L311, 8(f) NEXT 2): directions on a
    spherical spiral (z from +1 to -1, `turns` turns), each marched from ``centre`` to the offset
    surface like path_pivots, so consecutive pivots are neighbours (about 0.5 mm apart for 4096
    pivots on the head) except where the spiral crosses into another sheet of the surface."""
    out = np.empty((count, 3), dtype=np.float32)
    c = np.asarray(centre, dtype=np.float64)
    for k in range(count):
        z = 1.0 - 2.0 * (k + 0.5) / count
        phi = 2.0 * np.pi * turns * k / count
        rxy = np.sqrt(max(0.0, 1.0 - z * z))
        u = np.array([rxy * np.cos(phi), rxy * np.sin(phi), z])
        out[k] = _march_to_offset(model, params, u, offset, c)
    return out


@dataclass
class Config:
    """One synthetic workload (SURVEY.md 8(d) C1..C5 and small test variants)."""
    name: str
    model: str
    params: tuple
    lo: tuple
    size: float
    depth: int
    tool: tuple
    m: int
    n: int
    offset: float = 1.0
    fixed_pivots: tuple = ()
    centre: tuple = (0.0, 0.0, 0.0)
    note: str = ""

    def leaves(self):
        return octree_leaves(self.model, self.params, self.lo, self.size, self.depth)

    def min_half(self) -> float:
        return 0.5 * self.size / (1 << self.depth)

    def pivots(self, count: int, seed0: int = 1):
        fixed = [np.asarray(p, dtype=np.float32) for p in self.fixed_pivots]
        if count <= len(fixed):
            return np.stack(fixed[:count]) if count else np.zeros((0, 3), np.float32)
        # the pivot must also clear the voxel envelope: f <= 2 sqrt(3) h on any leaf point
        off = max(self.offset, 2.0 * np.sqrt(3.0) * self.min_half() + 0.05)
        extra = path_pivots(self.model, self.params, count - len(fixed), off, seed0, self.centre)
        return np.concatenate([np.stack(fixed) if fixed else np.zeros((0, 3), np.float32), extra])

    def toolpath(self, count: int, turns: float = 16.0):
        """`count` consecutive pivots of a continuous toolpath (toolpath_pivots)."""
        off = max(self.offset, 2.0 * np.sqrt(3.0) * self.min_half() + 0.05)
        return toolpath_pivots(self.model, self.params, count, off, self.centre, turns)

    def pivots_at(self, indices):
        """Pivots number k of the path for k in `indices` (pivots_at(range(n)) == pivots(n)):
        a rank of a pivot-sharded run generates only its own."""
        fixed = [np.asarray(p, dtype=np.float32) for p in self.fixed_pivots]
        off = max(self.offset, 2.0 * np.sqrt(3.0) * self.min_half() + 0.05)
        out = np.zeros((len(indices), 3), np.float32)
        for r, k in enumerate(indices):
            k = int(k)
            out[r] = fixed[k] if k < len(fixed) else path_pivots(self.model, self.params, 1, off,
                                                                   1 + k - len(fixed), self.centre)[0]
        return out


def _cfg(**kw):
    return Config(**kw)


CONFIGS = {
    # C1: 64^3 solid sphere (1 mm cells), single cylinder, 32x32, pivot on +z (analytic cap)
    "C1": _cfg(name="C1", model="sphere", params=(28.0,), lo=(-32.0, -32.0, -32.0), size=64.0,
               depth=6, tool=TOOL_1CYL, m=32, n=32, offset=3.0,
               fixed_pivots=((0.0, 0.0, 31.0), (9.0, -12.0, 27.5)),
               note="sphere Rs=28, 1 mm cells"),
    # C2: head-like, ~2M leaves, 3-cylinder tool, 64x64
    "C2": _cfg(name="C2", model="head", params=(), lo=(-56.0, -56.0, -56.0), size=112.0,
               depth=10, tool=TOOL_3CYL, m=64, n=64, note="head-like ~2M leaves"),
    # C3: head-like, ~27M leaves (paper's largest, 2048^3 class), 3-cylinder tool, 64x64
    "C3": _cfg(name="C3", model="head", params=(), lo=(-60.0, -60.0, -60.0), size=120.0,
               depth=12, tool=TOOL_3CYL, m=64, n=64, note="head-like ~27M leaves"),
    # C4: turbine-blade-like thin wall, ~10M leaves, 128x128
    "C4": _cfg(name="C4", model="blade", params=(), lo=(-71.0, -71.0, -51.0), size=142.0,
               depth=11, tool=TOOL_3CYL, m=128, n=128, centre=(0.0, 0.0, 10.0),
               note="twisted thin-wall blade on a hub ~10M leaves"),
    # C5: impeller-like, ~27M leaves, batch of pivots, 64x64
    "C5": _cfg(name="C5", model="impeller", params=(), lo=(-93.0, -93.0, -63.0), size=186.0,
               depth=11, tool=TOOL_3CYL, m=64, n=64, centre=(0.0, 0.0, 20.0),
               note="impeller hub + 14 swept blades ~27M leaves"),
    # small variants for parity tests (oracle finishes in seconds)
    "T_head": _cfg(name="T_head", model="head", params=(), lo=(-40.0, -40.0, -40.0), size=80.0,
                   depth=6, tool=TOOL_3CYL, m=64, n=64, note="head-like, 1.25 mm cells"),
    "T_head4": _cfg(name="T_head4", model="head", params=(), lo=(-40.0, -40.0, -40.0), size=80.0,
                    depth=6, tool=TOOL_PAPER4, m=48, n=40, note="head-like, paper 4-cyl tool, ragged grid"),
    "T_blade": _cfg(name="T_blade", model="blade", params=(), lo=(-72.0, -72.0, -52.0), size=144.0,
                    depth=7, tool=TOOL_3CYL, m=128, n=128, centre=(0.0, 0.0, 10.0),
                    note="blade, 1.1 mm cells, 128x128"),
    "T_imp": _cfg(name="T_imp", model="impeller", params=(), lo=(-64.0, -64.0, -34.0), size=128.0,
                  depth=7, tool=TOOL_3CYL, m=64, n=64, centre=(0.0, 0.0, 20.0),
                  note="impeller, 1 mm cells"),
}


def tool_arrays(tool):
    t = np.asarray(tool, dtype=np.float32).reshape(-1, 2)
    return t[:, 0].copy(), t[:, 1].copy()

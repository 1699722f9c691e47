"""fp64 CPU oracle for the accessibility map -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its
``cpu_baseline`` leg and ``--impl reference``) may import this package.  The
product path (``paper_conf_icpp_chenktkv19_b200``) never imports it and shares
no code with it.  See ``oracle.c`` for the definition it computes (PAPER.md
L86-88 problem statement, L97 CHECKBOX, Fig. 2 L60) and the 3-state margin.

Pins (tests/test_oracle.py): on-axis closed forms, cap/side contact closed
forms, an independent convex-QP distance, dense point sampling, the analytic
sphere cap, the single-voxel sphere sandwich (direction conventions),
symmetry, empty / enclosing / pivot-inside special cases and metamorphic
invariances.  No function here is "parity unpinned".
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None

DELTA = 1e-5  # rad, the north_star band (reading G10)


def build(force: bool = False) -> str:
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-shared", "-fPIC", src, "-o", _LIB, "-lm"])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        D = ctypes.POINTER(ctypes.c_double)
        F = ctypes.POINTER(ctypes.c_float)
        lib.oracle_axis_dist.restype = ctypes.c_double
        lib.oracle_axis_dist.argtypes = [D, ctypes.c_double, D, ctypes.c_double, ctypes.c_double]
        lib.oracle_box_cyl_hit.restype = ctypes.c_int
        lib.oracle_box_cyl_hit.argtypes = [D, ctypes.c_double, D, ctypes.c_double, ctypes.c_double,
                                           ctypes.c_double]
        lib.oracle_pair_state.restype = ctypes.c_int
        lib.oracle_pair_state.argtypes = [D, ctypes.c_double, D, D, D, ctypes.c_int, ctypes.c_double,
                                          ctypes.c_int]
        lib.oracle_cell_dir.restype = None
        lib.oracle_cell_dir.argtypes = [ctypes.c_int] * 4 + [D]
        lib.oracle_am_cells.restype = ctypes.c_int
        lib.oracle_am_cells.argtypes = [F, F, ctypes.c_int64, F, F, ctypes.c_int, F, ctypes.c_int,
                                        ctypes.c_int, ctypes.POINTER(ctypes.c_int64), ctypes.c_int64,
                                        ctypes.c_double, ctypes.c_int, ctypes.c_int,
                                        ctypes.POINTER(ctypes.c_uint8)]
        _lib = lib
    return _lib


def _d3(x):
    a = np.ascontiguousarray(np.asarray(x, dtype=np.float64).reshape(3))
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def axis_dist(v, h, d, z0, z1) -> float:
    """Distance from the tool axis line to box(v, h) cap slab [z0, z1]; -1 if empty."""
    lib = _load()
    va, vp = _d3(v)
    da, dp = _d3(d)
    return lib.oracle_axis_dist(vp, float(h), dp, float(z0), float(z1))


def box_cyl_hit(v, h, d, z0, z1, R) -> bool:
    lib = _load()
    va, vp = _d3(v)
    da, dp = _d3(d)
    return bool(lib.oracle_box_cyl_hit(vp, float(h), dp, float(z0), float(z1), float(R)))


def pair_state(v, h, d, tool, delta=DELTA, shortcuts=True) -> int:
    lib = _load()
    t = np.asarray(tool, dtype=np.float64).reshape(-1, 2)
    R = np.ascontiguousarray(t[:, 0])
    H = np.ascontiguousarray(t[:, 1])
    va, vp = _d3(v)
    da, dp = _d3(d)
    return lib.oracle_pair_state(vp, float(h), dp, R.ctypes.data_as(ctypes.POINTER(ctypes.c_double)),
                                 H.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), len(t),
                                 float(delta), int(bool(shortcuts)))


def cell_dir(i, j, m, n) -> np.ndarray:
    lib = _load()
    out = np.zeros(3, dtype=np.float64)
    lib.oracle_cell_dir(int(i), int(j), int(m), int(n), out.ctypes.data_as(ctypes.POINTER(ctypes.c_double)))
    return out


def am_states(centers, halfs, tool, pivot, m, n, cells=None, delta=DELTA, shortcuts=True,
              nthreads=0, return_threads=False):
    """3-state oracle AM.

    Returns uint8[m, n] (cells=None) or uint8[len(cells)] for flat cell indices
    ``cells`` (i * n + j): 2 robust collision, 0 robust clear, 1 band.
    """
    lib = _load()
    F = ctypes.POINTER(ctypes.c_float)
    c = np.ascontiguousarray(np.asarray(centers, dtype=np.float32).reshape(-1, 3))
    h = np.ascontiguousarray(np.asarray(halfs, dtype=np.float32).reshape(-1))
    t = np.asarray(tool, dtype=np.float32).reshape(-1, 2)
    R = np.ascontiguousarray(t[:, 0])
    H = np.ascontiguousarray(t[:, 1])
    p = np.ascontiguousarray(np.asarray(pivot, dtype=np.float32).reshape(3))
    if cells is None:
        cl = None
        ncell = m * n
        cptr = ctypes.POINTER(ctypes.c_int64)()
    else:
        cl = np.ascontiguousarray(np.asarray(cells, dtype=np.int64).reshape(-1))
        ncell = len(cl)
        cptr = cl.ctypes.data_as(ctypes.POINTER(ctypes.c_int64))
    out = np.zeros(ncell, dtype=np.uint8)
    used = lib.oracle_am_cells(c.ctypes.data_as(F), h.ctypes.data_as(F), len(h), R.ctypes.data_as(F),
                               H.ctypes.data_as(F), len(t), p.ctypes.data_as(F), int(m), int(n), cptr,
                               ncell, float(delta), int(bool(shortcuts)), int(nthreads),
                               out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8)))
    if used < 0:
        raise ValueError("too many cylinders for the oracle")
    res = out.reshape(m, n) if cells is None else out
    return (res, used) if return_threads else res


def pack_bits(am01: np.ndarray) -> np.ndarray:
    """Pack a {0,1}[m, n] map into the ABI layout: uint32[m, ceil(n/32)], LSB-first (reading G2)."""
    m, n = am01.shape
    W = (n + 31) // 32
    out = np.zeros((m, W), dtype=np.uint32)
    for j in range(n):
        out[:, j >> 5] |= (am01[:, j].astype(np.uint32) & 1) << np.uint32(j & 31)
    return out


def unpack_bits(words: np.ndarray, m: int, n: int) -> np.ndarray:
    """Inverse of pack_bits: uint32[m*ceil(n/32)] -> uint8[m, n]."""
    W = (n + 31) // 32
    w = np.asarray(words, dtype=np.uint32).reshape(m, W)
    j = np.arange(n)
    return ((w[:, j >> 5] >> (j & 31).astype(np.uint32)) & 1).astype(np.uint8)

"""ctypes binding of include/am.h (argument marshalling only).

Host data are numpy arrays; device data are ``torch`` CUDA tensors (PyTorch is
used for device memory and streams only).  Names follow the C ABI:
``am_create`` -> :class:`Context`, ``am_upload_voxels`` -> :meth:`Context.upload`,
``am_compute`` -> :meth:`Context.compute`, ``am_compute_batch`` ->
:meth:`Context.compute_batch`, ``am_compute_baseline`` ->
:meth:`Context.compute_baseline`.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# AM_LIBRARY: an alternative build of the same library (A/B experiments only)
LIB_PATH = os.environ.get("AM_LIBRARY") or os.path.join(_HERE, "libam.so")

AM_OK, AM_EINVAL, AM_ENOMEM, AM_ECUDA, AM_ESTATE = 0, -1, -2, -3, -4
OPT_GRID_CTAS, OPT_REFRESH_TILES, OPT_MORTON_SORT, OPT_BASELINE_REJECT, OPT_BAND_QUEUE = 1, 2, 3, 4, 5
K_COUNT = 20  # AM_K_COUNT (include/am.h)
SCHEME_PBOX, SCHEME_PBOX_AABB, SCHEME_PICA, SCHEME_MICA, SCHEME_AICA = 0, 1, 2, 3, 4  # AM_SCHEME_*
SCHEMES = {"pbox": 0, "pbox_aabb": 1, "pica": 2, "mica": 3, "aica": 4}
OPT_KERNEL_TIMING, OPT_PHASES, OPT_DIAG, OPT_CMAP_T, OPT_BRICKS, OPT_FUSED, OPT_BATCH = 6, 7, 8, 9, 10, 11, 12
OPT_BAND_SUBDIV, OPT_CMAP_T1, OPT_CMAP_ROWSCAN, OPT_CMAP_BRUTE, OPT_CMAP_BLOCK, OPT_MAP_CTAS, OPT_SUBBRICKS, OPT_BATCH_LANES, OPT_GRAPH = 13, 14, 15, 16, 17, 18, 19, 20, 21
OPT_L1_SAMPLE = 22
OPT_REUSE = 23
OPT_STAGE_FUSION = 24
OPT_STREAM_TMA = 25
OPT_PDL = 26
OPT_CMAP_FAR = 27
OPT_L1_SUBS = 28
OPT_LIVE_CAP = 29
OPT_L1_SPARSE = 30

# every symbol include/am.h declares
EXPORTS = ("am_create", "am_upload_voxels", "am_compute", "am_compute_batch", "am_compute_baseline",
           "am_set_option", "am_kernel_time", "am_kernel_stats", "am_kernel_name", "am_build_octree", "am_compute_octree", "am_unpack_cells", "am_pack_cells", "am_words_per_map",
           "am_num_voxels", "am_last_error", "am_destroy")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build the CUDA library first (python -c 'import __graft_entry__ as g; g.build()'). "
        "There is no CPU fallback.")


class _Cyl(ctypes.Structure):
    _fields_ = [("radius", ctypes.c_float), ("height", ctypes.c_float)]


class _Stats(ctypes.Structure):
    _fields_ = [(k, ctypes.c_int64) for k in (
        "voxels_streamed", "voxels_culled", "voxels_skipped", "voxels_live", "rows_rasterised",
        "band_pairs", "exact_tests", "exact_hits", "queue_overflow", "early_exit", "bricks_kept",
        "level_voxels", "rows_skipped_full")]


@dataclass
class Stats:
    voxels_streamed: int
    voxels_culled: int
    voxels_skipped: int
    voxels_live: int
    rows_rasterised: int
    band_pairs: int
    exact_tests: int
    exact_hits: int
    queue_overflow: int
    early_exit: int
    bricks_kept: int
    level_voxels: int
    rows_skipped_full: int


lib = ctypes.CDLL(LIB_PATH)
_P = ctypes.c_void_p
lib.am_create.restype = ctypes.c_int
lib.am_create.argtypes = [ctypes.POINTER(_Cyl), ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_int,
                          ctypes.POINTER(_P)]
lib.am_upload_voxels.restype = ctypes.c_int
lib.am_upload_voxels.argtypes = [_P, _P, _P, ctypes.c_int64, ctypes.c_int]
lib.am_compute.restype = ctypes.c_int
lib.am_compute.argtypes = [_P, ctypes.POINTER(ctypes.c_float), _P, ctypes.c_int, _P, ctypes.POINTER(_Stats)]
lib.am_compute_batch.restype = ctypes.c_int
lib.am_compute_batch.argtypes = [_P, ctypes.POINTER(ctypes.c_float), ctypes.c_int64, _P, ctypes.c_int, _P]
lib.am_compute_baseline.restype = ctypes.c_int
lib.am_compute_baseline.argtypes = [_P, ctypes.POINTER(ctypes.c_float), _P, ctypes.c_int, _P]
lib.am_set_option.restype = ctypes.c_int
lib.am_set_option.argtypes = [_P, ctypes.c_int, ctypes.c_int64]
lib.am_kernel_time.restype = ctypes.c_int
lib.am_kernel_time.argtypes = [_P, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int64)]
lib.am_kernel_stats.restype = ctypes.c_int
lib.am_kernel_stats.argtypes = [_P, ctypes.POINTER(ctypes.c_double), ctypes.POINTER(ctypes.c_int64)]
lib.am_build_octree.restype = ctypes.c_int
lib.am_build_octree.argtypes = [_P, ctypes.POINTER(ctypes.c_float), ctypes.c_float, ctypes.POINTER(ctypes.c_int64)]
lib.am_compute_octree.restype = ctypes.c_int
lib.am_compute_octree.argtypes = [_P, ctypes.POINTER(ctypes.c_float), ctypes.c_int, ctypes.c_int, ctypes.c_int, _P,
                                  ctypes.c_int, _P, ctypes.POINTER(ctypes.c_int64)]
lib.am_kernel_name.restype = ctypes.c_char_p
lib.am_kernel_name.argtypes = [ctypes.c_int]
lib.am_unpack_cells.restype = ctypes.c_int
lib.am_unpack_cells.argtypes = [_P, _P, _P, _P]
lib.am_pack_cells.restype = ctypes.c_int
lib.am_pack_cells.argtypes = [_P, _P, _P, _P]
lib.am_words_per_map.restype = ctypes.c_int
lib.am_words_per_map.argtypes = [_P]
lib.am_num_voxels.restype = ctypes.c_int64
lib.am_num_voxels.argtypes = [_P]
lib.am_last_error.restype = ctypes.c_char_p
lib.am_last_error.argtypes = [_P]
lib.am_destroy.restype = None
lib.am_destroy.argtypes = [_P]


KERNEL_NAMES = tuple(lib.am_kernel_name(k).decode() for k in range(K_COUNT))


def exported_symbols():
    """Names of include/am.h entry points found in libam.so."""
    return [s for s in EXPORTS if hasattr(lib, s)]


class AMError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"AM error {code}: {msg}")
        self.code = code


def words_per_map(m: int, n: int) -> int:
    return m * ((n + 31) // 32)


def unpack(words, m: int, n: int) -> np.ndarray:
    """uint32 words (ABI layout, include/am.h) -> uint8[m, n] collision map."""
    W = (n + 31) // 32
    w = np.asarray(words).view(np.uint32).reshape(m, W)
    j = np.arange(n)
    return ((w[:, j >> 5] >> (j & 31).astype(np.uint32)) & np.uint32(1)).astype(np.uint8)


def _is_torch_cuda(x):
    return hasattr(x, "is_cuda") and x.is_cuda


def _stream_handle(stream):
    if stream is None:
        return None
    if hasattr(stream, "cuda_stream"):
        return ctypes.c_void_p(stream.cuda_stream)
    return ctypes.c_void_p(int(stream))


def _check_out_dev(out, nwords: int, device: int):
    """A caller's device output: C-contiguous 4-byte elements on cuda:`device`, >= nwords."""
    if out.device.type != "cuda" or out.device.index != device:
        raise ValueError(f"out is on {out.device}, the context on cuda:{device}")
    if out.element_size() != 4 or out.dtype.is_floating_point:
        raise ValueError(f"out must hold 32-bit integer words (int32 / uint32), got {out.dtype}")
    if not out.is_contiguous():
        raise ValueError("out must be contiguous")
    if out.numel() < nwords:
        raise ValueError(f"out holds {out.numel()} words, the call writes {nwords}")


def _host_out(out, nwords: int):
    """A caller's host output as a writable C-contiguous 4-byte numpy view of >= nwords words."""
    if hasattr(out, "numpy") and not _is_torch_cuda(out):  # torch CPU tensor
        out = out.numpy()
    a = np.asarray(out)
    if a.dtype.itemsize != 4 or a.dtype.kind not in "iu":
        raise ValueError(f"out must hold 32-bit integer words (int32 / uint32), got {a.dtype}")
    if not a.flags["C_CONTIGUOUS"] or not a.flags["WRITEABLE"]:
        raise ValueError("out must be a writable C-contiguous array")
    if a.size < nwords:
        raise ValueError(f"out holds {a.size} words, the call writes {nwords}")
    return a


def _f3(p):
    a = np.ascontiguousarray(np.asarray(p, dtype=np.float32).reshape(3))
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_float))


class Context:
    """One am_ctx: a tool, an m x n orientation grid and a resident voxel model on one GPU."""

    def __init__(self, tool, m: int, n: int, device: int = 0):
        t = list(tool)
        arr = (_Cyl * max(len(t), 1))(*[_Cyl(float(r), float(h)) for r, h in t])
        h = _P()
        rc = lib.am_create(arr, len(t), int(m), int(n), int(device), ctypes.byref(h))
        if rc != AM_OK:
            raise AMError(rc, "am_create failed (tool / grid invalid or no usable CUDA device)")
        self._h = h
        self.m, self.n, self.device = int(m), int(n), int(device)
        self.words = lib.am_words_per_map(h)
        self.tool = tuple((float(r), float(hh)) for r, hh in t)

    # ------------------------------------------------------------------ helpers
    def _check(self, rc):
        if rc != AM_OK:
            raise AMError(rc, lib.am_last_error(self._h).decode())

    def close(self):
        if getattr(self, "_h", None):
            lib.am_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def set_option(self, key: int, value: int):
        self._check(lib.am_set_option(self._h, int(key), int(value)))

    def kernel_time(self):
        """am_kernel_time: (total ms, launches) of the streaming kernel since the last call."""
        ms = ctypes.c_double()
        n = ctypes.c_int64()
        self._check(lib.am_kernel_time(self._h, ctypes.byref(ms), ctypes.byref(n)))
        return ms.value, n.value

    def kernel_stats(self):
        """am_kernel_stats: {kernel name: (device ms, launches)} since the last call
        (ms only while OPT_KERNEL_TIMING = 2)."""
        ms = (ctypes.c_double * K_COUNT)()
        n = (ctypes.c_int64 * K_COUNT)()
        self._check(lib.am_kernel_stats(self._h, ms, n))
        return {KERNEL_NAMES[k]: (ms[k], n[k]) for k in range(K_COUNT)}

    def _dev_stream(self, t, stream):
        if not _is_torch_cuda(t):
            raise TypeError("expected a torch CUDA tensor")
        if stream is None:
            import torch
            stream = torch.cuda.current_stream(t.device)
        return _stream_handle(stream)

    def unpack_cells(self, words, cells, stream=None):
        """am_unpack_cells: device words (int32/uint32 [words]) -> device uint8 [m * n]."""
        _check_out_dev(words, self.words, self.device)
        if cells.numel() < self.m * self.n or cells.element_size() != 1 or not cells.is_contiguous():
            raise ValueError("cells must be a contiguous uint8 device tensor of >= m * n elements")
        self._check(lib.am_unpack_cells(self._h, _P(words.data_ptr()), _P(cells.data_ptr()),
                                        self._dev_stream(words, stream)))
        return cells

    def pack_cells(self, cells, words, stream=None):
        """am_pack_cells: device uint8 [m * n] -> device words."""
        _check_out_dev(words, self.words, self.device)
        if cells.numel() < self.m * self.n or cells.element_size() != 1 or not cells.is_contiguous():
            raise ValueError("cells must be a contiguous uint8 device tensor of >= m * n elements")
        self._check(lib.am_pack_cells(self._h, _P(cells.data_ptr()), _P(words.data_ptr()),
                                      self._dev_stream(cells, stream)))
        return words

    @property
    def num_voxels(self) -> int:
        return int(lib.am_num_voxels(self._h))

    # ------------------------------------------------------------------ calls
    def upload(self, centers, half_sizes):
        """am_upload_voxels: centres [N,3] + half sizes [N] (numpy host or torch CUDA float32)."""
        if _is_torch_cuda(centers):
            import torch
            if not _is_torch_cuda(half_sizes):
                raise ValueError("centres and half sizes must both be CUDA tensors (or both host arrays)")
            for name, t in (("centres", centers), ("half sizes", half_sizes)):
                if t.dtype != torch.float32:
                    raise ValueError(f"{name} must be float32, got {t.dtype}")
                if t.device.index != self.device:
                    raise ValueError(f"{name} are on {t.device}, the context on cuda:{self.device}")
            c = centers.contiguous()
            hs = half_sizes.contiguous()
            N = int(hs.numel())
            if c.numel() != 3 * N:
                raise ValueError(f"centres hold {c.numel()} floats, expected 3 x {N}")
            self._check(lib.am_upload_voxels(self._h, _P(c.data_ptr()), _P(hs.data_ptr()), N, 1))
        else:
            c = np.ascontiguousarray(np.asarray(centers, dtype=np.float32).reshape(-1, 3))
            hs = np.ascontiguousarray(np.asarray(half_sizes, dtype=np.float32).reshape(-1))
            if len(c) != len(hs):
                raise ValueError("centres and half sizes differ in length")
            self._check(lib.am_upload_voxels(self._h, _P(c.ctypes.data), _P(hs.ctypes.data), len(hs), 0))

    def compute(self, pivot, out=None, stream=None, stats: bool = False):
        """am_compute for one pivot.

        out=None -> host numpy uint32[words]; out = torch CUDA int32/uint32
        tensor of >= words elements -> written on the device (asynchronous on
        `stream`, default torch's current stream).  Returns (out, Stats|None).
        """
        _, pp = _f3(pivot)
        st = _Stats() if stats else None
        sp = ctypes.byref(st) if st is not None else None
        if out is not None and _is_torch_cuda(out):
            _check_out_dev(out, self.words, self.device)
            if stream is None:
                import torch
                stream = torch.cuda.current_stream(out.device)
            self._check(lib.am_compute(self._h, pp, _P(out.data_ptr()), 1, _stream_handle(stream), sp))
        else:
            if out is None:
                out = np.zeros(self.words, dtype=np.uint32)
            host = _host_out(out, self.words)
            self._check(lib.am_compute(self._h, pp, _P(host.ctypes.data), 0, _stream_handle(stream), sp))
        return out, (Stats(*[getattr(st, f[0]) for f in _Stats._fields_]) if st is not None else None)

    def compute_batch(self, pivots, out=None, stream=None):
        """am_compute_batch: P pivots -> P maps (host numpy uint32[P, words] or torch CUDA)."""
        pv = np.ascontiguousarray(np.asarray(pivots, dtype=np.float32).reshape(-1, 3))
        P = len(pv)
        pp = pv.ctypes.data_as(ctypes.POINTER(ctypes.c_float))
        if out is not None and _is_torch_cuda(out):
            _check_out_dev(out, P * self.words, self.device)
            if stream is None:
                import torch
                stream = torch.cuda.current_stream(out.device)
            self._check(lib.am_compute_batch(self._h, pp, P, _P(out.data_ptr()), 1, _stream_handle(stream)))
        else:
            if out is None:
                out = np.zeros((P, self.words), dtype=np.uint32)
            host = _host_out(out, P * self.words)
            self._check(lib.am_compute_batch(self._h, pp, P, _P(host.ctypes.data), 0, _stream_handle(stream)))
        return out

    def compute_baseline(self, pivot, out=None, stream=None):
        """am_compute_baseline: all-pairs exact test (PBox analogue)."""
        _, pp = _f3(pivot)
        if out is not None and _is_torch_cuda(out):
            _check_out_dev(out, self.words, self.device)
            if stream is None:
                import torch
                stream = torch.cuda.current_stream(out.device)
            self._check(lib.am_compute_baseline(self._h, pp, _P(out.data_ptr()), 1, _stream_handle(stream)))
        else:
            if out is None:
                out = np.zeros(self.words, dtype=np.uint32)
            host = _host_out(out, self.words)
            self._check(lib.am_compute_baseline(self._h, pp, _P(host.ctypes.data), 0, _stream_handle(stream)))
        return out

    def build_octree(self, root_lo, root_size) -> int:
        """am_build_octree: the octree of the resident leaves in the root cube; returns the node count."""
        _, lo = _f3(root_lo)
        n = ctypes.c_int64()
        self._check(lib.am_build_octree(self._h, lo, float(root_size), ctypes.byref(n)))
        return n.value

    def compute_octree(self, pivot, scheme, S=0, vdepth=0, out=None, stream=None, stats: bool = False):
        """am_compute_octree: the paper's orientation-per-thread scheme (SCHEMES name or
        AM_SCHEME_* value).  Returns (out, stats dict | None)."""
        sc = SCHEMES[scheme] if isinstance(scheme, str) else int(scheme)
        _, pp = _f3(pivot)
        st = (ctypes.c_int64 * 4)() if stats else None
        if out is not None and _is_torch_cuda(out):
            _check_out_dev(out, self.words, self.device)
            if stream is None:
                import torch
                stream = torch.cuda.current_stream(out.device)
            self._check(lib.am_compute_octree(self._h, pp, sc, int(S), int(vdepth), _P(out.data_ptr()), 1,
                                              _stream_handle(stream), st))
        else:
            if out is None:
                out = np.zeros(self.words, dtype=np.uint32)
            host = _host_out(out, self.words)
            self._check(lib.am_compute_octree(self._h, pp, sc, int(S), int(vdepth), _P(host.ctypes.data), 0,
                                              _stream_handle(stream), st))
        sd = None
        if st is not None:
            sd = {"nodes_popped": st[0], "box_tests": st[1], "ica_evals": st[2], "max_popped_per_thread": st[3]}
        return out, sd

    def am(self, pivot) -> np.ndarray:
        """Convenience: uint8[m, n] AICA map of one pivot (host)."""
        w, _ = self.compute(pivot)
        return unpack(w, self.m, self.n)

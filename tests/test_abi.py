"""The C-ABI library loads and exports every symbol include/am.h declares (CPU, no compute)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def am():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icpp_chenktkv19_b200 as am
    return am


def _declared():
    src = open(os.path.join(ROOT, "include", "am.h")).read()
    return sorted(set(re.findall(r"\b(am_[a-z_]+)\s*\(", src)))


def test_header_symbols_exported(am):
    declared = _declared()
    assert len(declared) == 17
    lib = ctypes.CDLL(am.LIB_PATH)
    for s in declared:
        assert hasattr(lib, s), s
    assert sorted(am.binding.EXPORTS) == declared


def test_library_targets_sm100a(am):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", am.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_argument_validation_without_gpu(am):
    lib = am.lib
    Cyl = am.binding._Cyl
    h = ctypes.c_void_p()
    good = (Cyl * 1)(Cyl(6.35, 25.4))
    bad_r = (Cyl * 1)(Cyl(-1.0, 25.4))
    bad_h = (Cyl * 1)(Cyl(1.0, float("nan")))
    assert lib.am_create(good, 0, 8, 8, 0, ctypes.byref(h)) == am.AM_EINVAL
    assert lib.am_create(good, 9, 8, 8, 0, ctypes.byref(h)) == am.AM_EINVAL
    assert lib.am_create(bad_r, 1, 8, 8, 0, ctypes.byref(h)) == am.AM_EINVAL
    assert lib.am_create(bad_h, 1, 8, 8, 0, ctypes.byref(h)) == am.AM_EINVAL
    assert lib.am_create(good, 1, 0, 8, 0, ctypes.byref(h)) == am.AM_EINVAL
    assert lib.am_create(good, 1, 8, 1025, 0, ctypes.byref(h)) == am.AM_EINVAL
    assert lib.am_create(good, 1, 8, 8, 0, None) == am.AM_EINVAL
    # NULL-context calls
    assert lib.am_words_per_map(None) == -1
    assert lib.am_num_voxels(None) == -1
    assert lib.am_upload_voxels(None, None, None, 0, 0) == am.AM_EINVAL
    assert lib.am_compute(None, None, None, 0, None, None) == am.AM_EINVAL
    assert lib.am_compute_batch(None, None, 0, None, 0, None) == am.AM_EINVAL
    assert lib.am_compute_baseline(None, None, None, 0, None) == am.AM_EINVAL
    assert lib.am_set_option(None, 1, 0) == am.AM_EINVAL
    assert lib.am_kernel_time(None, None, None) == am.AM_EINVAL
    assert lib.am_kernel_stats(None, None, None) == am.AM_EINVAL
    assert lib.am_build_octree(None, None, 1.0, None) == am.AM_EINVAL
    assert lib.am_compute_octree(None, None, 0, 0, 0, None, 0, None, None) == am.AM_EINVAL
    assert lib.am_unpack_cells(None, None, None, None) == am.AM_EINVAL
    assert lib.am_pack_cells(None, None, None, None) == am.AM_EINVAL
    assert lib.am_last_error(None) == b"NULL context"
    lib.am_destroy(None)


def test_unpack_layout(am):
    import numpy as np
    words = np.array([0b101, 1, 0x80000000, 0], dtype=np.uint32)  # m=2, n=40 -> W=2
    u = am.unpack(words, 2, 40)
    assert u[0, 0] == 1 and u[0, 1] == 0 and u[0, 2] == 1 and u[0, 31] == 0
    assert u[0, 32] == 1  # row 0, word 1, bit 0
    assert u[1, 31] == 1 and u.sum() == 4


def test_kernel_names_match_header(am):
    """binding.K_COUNT / KERNEL_NAMES mirror the AM_K_* enum of include/am.h."""
    src = open(os.path.join(ROOT, "include", "am.h")).read()
    body = src[src.index("AM_K_L0_CONES = 0"):src.index("AM_K_COUNT")]
    names = re.findall(r"\b(AM_K_[A-Z0-9_]+)\b", body)
    assert len(names) == am.binding.K_COUNT
    assert len(set(am.binding.KERNEL_NAMES)) == am.binding.K_COUNT
    assert am.lib.am_kernel_name(am.binding.K_COUNT) is None
    assert am.lib.am_kernel_name(-1) is None


def test_option_keys_match_header(am):
    """Every AM_OPT_* key of include/am.h has the same value in the binding (OPT_*), and the
    binding defines no key the header lacks."""
    src = open(os.path.join(ROOT, "include", "am.h")).read()
    header = {k[len("AM_OPT_"):]: int(v)
              for k, v in re.findall(r"^\s*(AM_OPT_[A-Z0-9_]+)\s*=\s*(\d+)\s*,?\s*/\*", src, re.M)}
    binding = {k[len("OPT_"):]: getattr(am.binding, k) for k in dir(am.binding) if k.startswith("OPT_")}
    assert header == binding
    assert sorted(header.values()) == list(range(1, len(header) + 1))

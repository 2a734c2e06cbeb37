"""C-ABI boundary tests that need no GPU: the library loads, exports every
symbol include/eggsync.h declares, and argument validation returns the
documented codes before touching any device or output buffer."""
import ctypes
import os
import re

import numpy as np
import pytest

from paper_conf_edbt_jorgensena23_b200 import eggsync as E

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "eggsync.h")


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(eggsync_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    L = E.lib()
    names = _declared()
    assert len(names) >= 20
    for nm in names:
        assert hasattr(L, nm), nm
    assert sorted(E.SYMBOLS) == names


def test_library_is_sm100a_and_has_no_host_fallback():
    out = os.popen(f"/usr/local/cuda/bin/cuobjdump --list-elf {E.LIB_PATH} 2>&1").read()
    assert "sm_100a" in out
    assert E.lib().eggsync_version().decode().endswith("(sm_100a)")


def test_default_opts():
    o = E.default_opts()
    assert o.struct_size == ctypes.sizeof(E.Opts)
    assert o.max_iters == 10000 and o.device == -1 and o.device_pointers == 0
    assert o.cw_factor == 1.0


@pytest.mark.parametrize("n,d,eps", [(0, 2, 0.05), (10, 0, 0.05), (10, 33, 0.05), (10, 2, 0.0),
                                     (10, 2, float("nan")), (10, 2, float("inf")), (10, 2, -1.0),
                                     (2 ** 31, 2, 0.05), (10, 32, 1e-7)])
def test_invalid_arguments_return_einval_and_leave_outputs(n, d, eps):
    pts = np.full((2, 2), 0.5, np.float32)
    lab = np.full(2, -7, np.int32)
    it = ctypes.c_int32(-9)
    rc = E.lib().eggsync_cluster(pts.ctypes.data_as(ctypes.c_void_p), n, d, ctypes.c_float(eps),
                                 lab.ctypes.data_as(ctypes.c_void_p), ctypes.byref(it))
    assert rc == E.EINVAL, E.last_error()
    assert (lab == -7).all() and it.value == -9
    assert E.last_error()


def test_null_pointers_are_einval():
    L = E.lib()
    it = ctypes.c_int32(0)
    assert L.eggsync_cluster(None, 10, 2, ctypes.c_float(0.05), None, ctypes.byref(it)) == E.EINVAL
    lab = np.zeros(10, np.int32)
    pts = np.zeros((10, 2), np.float32)
    assert L.eggsync_cluster(pts.ctypes.data_as(ctypes.c_void_p), 10, 2, ctypes.c_float(0.05), None,
                             ctypes.byref(it)) == E.EINVAL
    assert L.eggsync_step(None, 10, 2, ctypes.c_float(0.05), None) == E.EINVAL


def test_bad_opts_struct_size():
    o = E.default_opts()
    o.struct_size = 3
    pts = np.zeros((4, 2), np.float32)
    lab = np.zeros(4, np.int32)
    it = ctypes.c_int32(0)
    rc = E.lib().eggsync_cluster_ex(pts.ctypes.data_as(ctypes.c_void_p), 4, 2, ctypes.c_float(0.05),
                                    ctypes.byref(o), lab.ctypes.data_as(ctypes.c_void_p), ctypes.byref(it))
    assert rc == E.EINVAL


def test_no_cpu_fallback_without_device(cuda_available):
    if cuda_available:
        pytest.skip("device present")
    with pytest.raises(E.EggSyncError) as ei:
        E.cluster(np.full((8, 2), 0.5, np.float32), 0.05)
    assert ei.value.rc == E.ECUDA
    assert "no CUDA device" in str(ei.value)


@pytest.mark.parametrize("n,d,eps", [(0, 2, 0.05), (10, 0, 0.05), (10, 33, 0.05), (10, 2, 0.0),
                                     (10, 2, float("nan")), (2 ** 31, 2, 0.05)])
def test_sync_entry_points_validate_before_touching_outputs(n, d, eps):
    """eggsync_sync_step / eggsync_sync_lambda (F4) reject bad sizes with EINVAL, outputs untouched."""
    pts = np.full((2, 2), 0.5, np.float32)
    rc = ctypes.c_double(-3.0)
    it = ctypes.c_int32(-9)
    L = E.lib()
    assert L.eggsync_sync_step(pts.ctypes.data_as(ctypes.c_void_p), n, d, ctypes.c_float(eps), 0,
                               ctypes.byref(rc), None) == E.EINVAL
    assert L.eggsync_sync_lambda(pts.ctypes.data_as(ctypes.c_void_p), n, d, ctypes.c_float(eps),
                                 ctypes.c_double(0.999), 10, 0, ctypes.byref(it), ctypes.byref(rc)) == E.EINVAL
    assert rc.value == -3.0 and it.value == -9 and (pts == 0.5).all()
    assert L.eggsync_sync_step(None, 10, 2, ctypes.c_float(0.05), 0, None, None) == E.EINVAL


def test_sync_lambda_rejects_bad_loop_arguments(cuda_available):
    if cuda_available:
        pytest.skip("device present: covered by the GPU tests")
    pts = np.full((4, 2), 0.5, np.float32)
    # without a device the call fails loudly (no CPU fallback) before the loop arguments matter
    with pytest.raises(E.EggSyncError) as ei:
        E.sync_step(pts, 0.05)
    assert ei.value.rc == E.ECUDA


@pytest.mark.parametrize("f", [0.0, -0.5, 1.0000001, float("nan"), float("inf")])
def test_cw_factor_out_of_range_is_einval(f):
    """opts.cw_factor must lie in (0, 1] (c_w <= eps/(2 sqrt d), L252); checked before any output."""
    o = E.default_opts()
    o.cw_factor = f
    pts = np.full((4, 2), 0.5, np.float32)
    lab = np.full(4, -7, np.int32)
    it = ctypes.c_int32(-9)
    rc = E.lib().eggsync_cluster_ex(pts.ctypes.data_as(ctypes.c_void_p), 4, 2, ctypes.c_float(0.05),
                                    ctypes.byref(o), lab.ctypes.data_as(ctypes.c_void_p), ctypes.byref(it))
    assert rc == E.EINVAL and "cw_factor" in E.last_error()
    assert (lab == -7).all() and it.value == -9


def test_term_mode_validation():
    """term_mode: GRID (0), DEF42 (1) or DEF42_DIRECT (2), the last two cluster_ex only; anything
    else EINVAL before any output."""
    pts = np.full((4, 2), 0.5, np.float32)
    lab = np.full(4, -7, np.int32)
    it = ctypes.c_int32(-9)
    o = E.default_opts()
    o.term_mode = 3
    rc = E.lib().eggsync_cluster_ex(pts.ctypes.data_as(ctypes.c_void_p), 4, 2, ctypes.c_float(0.05),
                                    ctypes.byref(o), lab.ctypes.data_as(ctypes.c_void_p), ctypes.byref(it))
    assert rc == E.EINVAL and (lab == -7).all() and it.value == -9
    o.term_mode = E.TERM_DEF42
    f1, f2 = ctypes.c_int32(-3), ctypes.c_int32(-3)
    rc = E.lib().eggsync_step_ex(pts.ctypes.data_as(ctypes.c_void_p), 4, 2, ctypes.c_float(0.05), ctypes.byref(o),
                                 ctypes.byref(f1), ctypes.byref(f2))
    assert rc == E.EINVAL and f1.value == -3 and (pts == 0.5).all()

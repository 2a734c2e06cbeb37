"""ctypes wrapper of the fp64 CPU oracle (oracle/oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, ``__graft_entry__.smoke()`` and
bench.py's ``cpu_baseline`` / ``--impl reference`` legs.  The product package
``paper_conf_edbt_jorgensena23_b200`` never imports this module, and this
module imports nothing from the product package.

Every function follows PAPER.md; see the header of oracle.c for the passages
and the readings (R1..R14) it implements.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")

OK, NOT_CONVERGED, EINVAL, ENOMEM, EPARTITION = 0, 1, -1, -3, -6
GRID, DEF42 = 0, 1


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (fp64, -ffp-contract=off, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-ffp-contract=off", "-fno-fast-math", "-fopenmp",
                               "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        i64, i32, f32 = ctypes.c_int64, ctypes.c_int32, ctypes.c_float
        vp = ctypes.c_void_p
        L.oracle_constants.argtypes = [f32, i32, vp]
        L.oracle_constants.restype = None
        f64 = ctypes.c_double
        L.oracle_constants_cw.argtypes = [f32, i32, f64, vp]
        L.oracle_constants_cw.restype = None
        L.oracle_step.argtypes = [vp, i64, i32, f32, vp, vp, vp, i32]
        L.oracle_step.restype = ctypes.c_int
        L.oracle_step_cw.argtypes = [vp, i64, i32, f32, f64, vp, vp, vp, i32]
        L.oracle_step_cw.restype = ctypes.c_int
        L.oracle_cluster.argtypes = [vp, i64, i32, f32, i32, i32, vp, vp, vp, vp]
        L.oracle_cluster.restype = ctypes.c_int
        L.oracle_cluster_cw.argtypes = [vp, i64, i32, f32, f64, i32, i32, vp, vp, vp, vp]
        L.oracle_cluster_cw.restype = ctypes.c_int
        L.oracle_step_sample.argtypes = [vp, i64, i32, f32, vp, i64, vp, vp]
        L.oracle_step_sample.restype = ctypes.c_int
        L.oracle_terminal_sample.argtypes = [vp, i64, i32, f32, vp, vp, i64]
        L.oracle_terminal_sample.restype = ctypes.c_int64
        L.oracle_order_parameter.argtypes = [vp, i64, i32, f32, vp, vp]
        L.oracle_order_parameter.restype = ctypes.c_int
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def constants(eps: float, d: int, cw_factor: float = 1.0) -> dict:
    """eps, eps^2, c_w (L252, times cw_factor), 1/c_w, w (Eq.4), delta (L110), (eps+delta)^2."""
    out = np.zeros(7, np.float64)
    lib().oracle_constants_cw(ctypes.c_float(eps), d, cw_factor, _p(out))
    keys = ["eps", "eps2", "cw", "inv_cw", "w", "delta", "ed2"]
    return dict(zip(keys, out.tolist()))


def step(X, eps: float, compute_f2: bool = False, cw_factor: float = 1.0):
    """One Eq.1 update of the state X (n x d; fp32 or fp64, converted to fp64).

    Returns (Xn fp64, nbr int32, flags) with flags = (F1_grid, F1_def42, F2);
    F2 is -1 when not evaluated (neither first-term form holds and not compute_f2).
    """
    X = np.ascontiguousarray(X, dtype=np.float64)
    n, d = X.shape
    Xn = np.empty_like(X)
    nbr = np.empty(n, np.int32)
    flags = np.zeros(3, np.int32)
    rc = lib().oracle_step_cw(_p(X), n, d, ctypes.c_float(eps), cw_factor, _p(Xn), _p(nbr), _p(flags),
                              int(compute_f2))
    if rc != OK:
        raise RuntimeError(f"oracle_step rc={rc}")
    return Xn, nbr, tuple(int(f) for f in flags)


def order_parameter(X, eps: float):
    """Cluster order parameter r_c of the state X (Eq.2, Alg 1 l.6 L54).

    Returns (r_c, per-point inner means) in fp64.
    """
    X = np.ascontiguousarray(X, dtype=np.float64)
    n, d = X.shape
    out = np.zeros(1, np.float64)
    rcp = np.empty(n, np.float64)
    rc = lib().oracle_order_parameter(_p(X), n, d, ctypes.c_float(eps), _p(out), _p(rcp))
    if rc != OK:
        raise RuntimeError(f"oracle_order_parameter rc={rc}")
    return float(out[0]), rcp


def cluster(X32, eps: float, term_mode: int = GRID, max_iters: int = 10000, cw_factor: float = 1.0):
    """Full clustering by the definition.  Returns dict(rc, X, labels, iters, cell_labels)."""
    X32 = np.ascontiguousarray(X32, dtype=np.float32)
    n, d = X32.shape
    Xo = np.empty((n, d), np.float64)
    labels = np.empty(n, np.int32)
    cells = np.empty(n, np.int32)
    iters = np.zeros(1, np.int32)
    rc = lib().oracle_cluster_cw(_p(X32), n, d, ctypes.c_float(eps), cw_factor, term_mode, max_iters,
                                 _p(Xo), _p(labels), _p(iters), _p(cells))
    if rc < 0 and rc != EPARTITION:
        raise RuntimeError(f"oracle_cluster rc={rc}")
    return {"rc": rc, "X": Xo, "labels": labels, "iters": int(iters[0]), "cell_labels": cells}


def step_sample(X32, eps: float, idx):
    """Eq.1 update of the sampled points idx against the full float32 state."""
    X32 = np.ascontiguousarray(X32, dtype=np.float32)
    n, d = X32.shape
    idx = np.ascontiguousarray(idx, dtype=np.int64)
    m = idx.shape[0]
    Xn = np.empty((m, d), np.float64)
    nbr = np.empty(m, np.int32)
    rc = lib().oracle_step_sample(_p(X32), n, d, ctypes.c_float(eps), _p(idx), m, _p(Xn), _p(nbr))
    if rc != OK:
        raise RuntimeError(f"oracle_step_sample rc={rc}")
    return Xn, nbr


def terminal_violations(X32, eps: float, labels, idx) -> int:
    """Theorem 4.7 check on sampled points: #pairs where (same label) != (within eps)."""
    X32 = np.ascontiguousarray(X32, dtype=np.float32)
    n, d = X32.shape
    labels = np.ascontiguousarray(labels, dtype=np.int32)
    idx = np.ascontiguousarray(idx, dtype=np.int64)
    v = lib().oracle_terminal_sample(_p(X32), n, d, ctypes.c_float(eps), _p(labels), _p(idx),
                                     idx.shape[0])
    if v < 0:
        raise RuntimeError("oracle_terminal_sample failed")
    return int(v)

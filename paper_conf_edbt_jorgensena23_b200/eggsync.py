"""Thin ctypes binding of libeggsync.so (include/eggsync.h).

Argument marshalling only: every step of the method runs in the library's
CUDA kernels.  Host inputs are numpy arrays; device inputs are CUDA torch
tensors (their data pointers are passed with ``device_pointers=1``).  There
is no CPU fallback -- if the library or a CUDA device is missing, calls raise.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("EGGSYNC_LIB") or os.path.join(_HERE, "libeggsync.so")

OK, NOT_CONVERGED, EINVAL, EDOMAIN, ENOMEM, ECUDA, ENCCL = 0, 1, -1, -2, -3, -4, -5
MAX_D = 32

#: every symbol include/eggsync.h declares
SYMBOLS = [
    "eggsync_default_opts", "eggsync_cluster", "eggsync_cluster_ex", "eggsync_step", "eggsync_step_ex",
    "eggsync_last_error", "eggsync_version", "eggsync_ctx_create", "eggsync_ctx_destroy",
    "eggsync_ctx_load", "eggsync_ctx_build", "eggsync_ctx_update", "eggsync_ctx_second_term",
    "eggsync_ctx_flags", "eggsync_ctx_cur_coords", "eggsync_ctx_next_coords", "eggsync_ctx_pack",
    "eggsync_ctx_unpack", "eggsync_ctx_advance", "eggsync_ctx_labels", "eggsync_ctx_coords",
    "eggsync_ctx_run", "eggsync_ctx_stream", "eggsync_ctx_work", "eggsync_ctx_tc_work", "eggsync_ctx_launches",
    "eggsync_release_cache", "eggsync_ctx_update_owned", "eggsync_ctx_owned_count", "eggsync_ctx_pack_owned",
    "eggsync_ctx_unpack_owned", "eggsync_ctx_plan_owned", "eggsync_ctx_update_planned", "eggsync_ctx_set_own", "eggsync_sync_step",
    "eggsync_sync_lambda",
]


class EggSyncError(RuntimeError):
    def __init__(self, rc: int, msg: str):
        super().__init__(f"eggsync error {rc}: {msg}")
        self.rc = rc


class Stats(ctypes.Structure):
    """eggsync_stats: Table 1 columns (L364-371) + counters."""
    _fields_ = [("t_alloc", ctypes.c_double), ("t_build", ctypes.c_double), ("t_update", ctypes.c_double),
                ("t_extra_check", ctypes.c_double), ("t_cluster", ctypes.c_double),
                ("t_free", ctypes.c_double), ("t_transfer", ctypes.c_double), ("iters", ctypes.c_int32),
                ("n_cells_first", ctypes.c_int32), ("n_cells_last", ctypes.c_int32),
                ("sort_skipped", ctypes.c_int32), ("device_bytes", ctypes.c_int64)]

    def as_dict(self):
        return {k: getattr(self, k) for k, _ in self._fields_}


class Opts(ctypes.Structure):
    _fields_ = [("struct_size", ctypes.c_int32), ("max_iters", ctypes.c_int32), ("device", ctypes.c_int32),
                ("device_pointers", ctypes.c_int32), ("stream", ctypes.c_void_p), ("term_mode", ctypes.c_int32),
                ("coords_out", ctypes.c_void_p), ("nbr_count_out", ctypes.c_void_p),
                ("stats", ctypes.POINTER(Stats)), ("cw_factor", ctypes.c_double)]


_lib = None


def lib():
    """Load the CUDA library; fail loudly if it has not been built (no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
        L = ctypes.CDLL(LIB_PATH)
        vp, i64, i32, f32 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_float
        sig = {
            "eggsync_default_opts": ([vp], None),
            "eggsync_cluster": ([vp, i64, i32, f32, vp, vp], ctypes.c_int),
            "eggsync_cluster_ex": ([vp, i64, i32, f32, vp, vp, vp], ctypes.c_int),
            "eggsync_step": ([vp, i64, i32, f32, vp], ctypes.c_int),
            "eggsync_step_ex": ([vp, i64, i32, f32, vp, vp, vp], ctypes.c_int),
            "eggsync_last_error": ([], ctypes.c_char_p),
            "eggsync_version": ([], ctypes.c_char_p),
            "eggsync_ctx_create": ([i64, i32, f32, i32, vp, ctypes.POINTER(vp)], ctypes.c_int),
            "eggsync_ctx_destroy": ([vp], None),
            "eggsync_ctx_load": ([vp, vp, i32], ctypes.c_int),
            "eggsync_ctx_build": ([vp, vp], ctypes.c_int),
            "eggsync_ctx_update": ([vp, i64, i64], ctypes.c_int),
            "eggsync_ctx_second_term": ([vp, i64, i64], ctypes.c_int),
            "eggsync_ctx_flags": ([vp, vp, vp], ctypes.c_int),
            "eggsync_ctx_cur_coords": ([vp], vp),
            "eggsync_ctx_next_coords": ([vp], vp),
            "eggsync_ctx_pack": ([vp, i64, i64, vp], ctypes.c_int),
            "eggsync_ctx_unpack": ([vp, vp, i32, i64], ctypes.c_int),
            "eggsync_ctx_advance": ([vp], ctypes.c_int),
            "eggsync_ctx_labels": ([vp, vp, i32], ctypes.c_int),
            "eggsync_ctx_coords": ([vp, vp, i32], ctypes.c_int),
            "eggsync_ctx_run": ([vp, i32, vp], ctypes.c_int),
            "eggsync_ctx_stream": ([vp], vp),
            "eggsync_ctx_work": ([vp, i32, vp], ctypes.c_int),
            "eggsync_ctx_tc_work": ([vp, i32, vp], ctypes.c_int),
            "eggsync_ctx_launches": ([vp], ctypes.c_int64),
            "eggsync_release_cache": ([], None),
            "eggsync_ctx_update_owned": ([vp, i32, i32], ctypes.c_int),
            "eggsync_ctx_owned_count": ([vp, i32], ctypes.c_int64),
            "eggsync_ctx_pack_owned": ([vp, i32, i32, vp], ctypes.c_int),
            "eggsync_ctx_unpack_owned": ([vp, vp, i32], ctypes.c_int),
            "eggsync_ctx_plan_owned": ([vp, i32, i32, vp], ctypes.c_int),
            "eggsync_ctx_update_planned": ([vp, i32, i32, vp], ctypes.c_int),
            "eggsync_ctx_set_own": ([vp, i64], ctypes.c_int),
            "eggsync_sync_step": ([vp, i64, i32, f32, i32, vp, vp], ctypes.c_int),
            "eggsync_sync_lambda": ([vp, i64, i32, f32, ctypes.c_double, i32, i32, vp, vp], ctypes.c_int),
        }
        for name, (args, res) in sig.items():
            fn = getattr(L, name)
            fn.argtypes = args
            fn.restype = res
        _lib = L
    return _lib


def release_cache() -> None:
    """Free the library's cached device workspaces."""
    lib().eggsync_release_cache()


def last_error() -> str:
    return lib().eggsync_last_error().decode()


def _check(rc: int, allow=(OK,)):
    if rc not in allow:
        raise EggSyncError(rc, last_error())
    return rc


def _is_torch_cuda(x):
    return type(x).__module__.startswith("torch") and getattr(x, "is_cuda", False)


#: cudaStreamLegacy: the legacy default stream as an explicit handle (a NULL handle would
#: ask the library for its own non-blocking stream, unordered with the caller's work)
_STREAM_LEGACY = 1


def _stream_arg(handle: int):
    """A torch stream handle for the C ABI: torch's default stream (0) becomes cudaStreamLegacy,
    so the library's work is ordered after the kernels / copies that produced the tensors."""
    return ctypes.c_void_p(int(handle) or _STREAM_LEGACY)


def _ptr(a):
    if _is_torch_cuda(a):
        return ctypes.c_void_p(a.data_ptr())
    return a.ctypes.data_as(ctypes.c_void_p)


def default_opts() -> Opts:
    o = Opts()
    lib().eggsync_default_opts(ctypes.byref(o))
    return o


def _host_points(points, writable=False):
    a = np.ascontiguousarray(points, dtype=np.float32)
    if a.ndim != 2:
        raise ValueError("points must be (n, d)")
    return a.copy() if writable else a  # step() writes D^{t+1}: never alias the caller's array


TERM_GRID, TERM_DEF42, TERM_DEF42_DIRECT = 0, 1, 2


def cluster(points, eps: float, *, max_iters: int = 10000, coords: bool = False, stats: bool = False,
            stream=None, cw_factor: float = 1.0, term_mode: int = TERM_GRID):
    """EGG-SynC clustering (Alg 4).  points: (n,d) float32 numpy (host) or CUDA torch tensor.

    Returns dict(labels, iters, converged[, coords][, stats]).  Device inputs give device outputs.
    """
    dev = _is_torch_cuda(points)
    o = default_opts()
    o.max_iters = max_iters
    o.cw_factor = cw_factor
    o.term_mode = term_mode
    if dev:
        import torch
        assert points.dtype == torch.float32 and points.is_contiguous() and points.dim() == 2
        n, d = points.shape
        o.device_pointers = 1
        o.device = points.device.index
        o.stream = _stream_arg(stream if stream is not None else torch.cuda.current_stream(points.device).cuda_stream)
        labels = torch.empty(n, dtype=torch.int32, device=points.device)
        co = torch.empty((n, d), dtype=torch.float32, device=points.device) if coords else None
    else:
        points = _host_points(points)
        n, d = points.shape
        labels = np.empty(n, np.int32)
        co = np.empty((n, d), np.float32) if coords else None
    st = Stats()
    if stats:
        o.stats = ctypes.pointer(st)
    if co is not None:
        o.coords_out = _ptr(co)
    iters = ctypes.c_int32(0)
    rc = lib().eggsync_cluster_ex(_ptr(points), n, d, ctypes.c_float(eps), ctypes.byref(o), _ptr(labels),
                                  ctypes.byref(iters))
    _check(rc, (OK, NOT_CONVERGED))
    out = {"labels": labels, "iters": iters.value, "converged": rc == OK}
    if coords:
        out["coords"] = co
    if stats:
        out["stats"] = st.as_dict()
    return out


def step(points, eps: float, *, nbr: bool = False, cw_factor: float = 1.0):
    """One Eq.1 update (eggsync_step_ex) of host points.  Returns dict(points, first, second, synced[, nbr])."""
    x = _host_points(points, writable=True)
    n, d = x.shape
    o = default_opts()
    o.cw_factor = cw_factor
    cnt = np.empty(n, np.int32) if nbr else None
    if nbr:
        o.nbr_count_out = _ptr(cnt)
    f1, f2 = ctypes.c_int32(0), ctypes.c_int32(0)
    _check(lib().eggsync_step_ex(_ptr(x), n, d, ctypes.c_float(eps), ctypes.byref(o), ctypes.byref(f1),
                                 ctypes.byref(f2)))
    out = {"points": x, "first": f1.value, "second": f2.value, "synced": int(f1.value == 1 and f2.value == 1)}
    if nbr:
        out["nbr"] = cnt
    return out


def _sync_points(points):
    """(array to pass, n, d, on_device): device tensors in place, host arrays copied (never aliased).

    The direct-path entry points run on the legacy default stream of the current device:
    a device tensor's device becomes current and its producer stream is drained first.
    """
    if _is_torch_cuda(points):
        import torch
        assert points.dtype == torch.float32 and points.is_contiguous() and points.dim() == 2
        torch.cuda.set_device(points.device)
        torch.cuda.current_stream(points.device).synchronize()
        return points, points.shape[0], points.shape[1], 1
    x = _host_points(points, writable=True)
    return x, x.shape[0], x.shape[1], 0


def sync_step(points, eps: float, *, nbr: bool = False):
    """Direct (GPU-SynC-style, no grid) Eq.1 update + Eq.2 r_c of the input (eggsync_sync_step).

    Host numpy input: returns a new array; CUDA tensor input: updated in place.
    Returns dict(points, rc[, nbr]).
    """
    x, n, d, dev = _sync_points(points)
    cnt = None
    if nbr:
        if dev:
            import torch
            cnt = torch.empty(n, dtype=torch.int32, device=x.device)
        else:
            cnt = np.empty(n, np.int32)
    rc = ctypes.c_double(0.0)
    _check(lib().eggsync_sync_step(_ptr(x), n, d, ctypes.c_float(eps), dev, ctypes.byref(rc),
                                   _ptr(cnt) if nbr else None))
    out = {"points": x, "rc": rc.value}
    if nbr:
        out["nbr"] = cnt
    return out


def sync_lambda(points, eps: float, lam: float = 0.999, *, max_iters: int = 10000):
    """SynC with lambda-termination (Alg 1) on the GPU (eggsync_sync_lambda).

    Returns dict(points, iters, rc, reached) -- reached is False when max_iters stopped it.
    """
    x, n, d, dev = _sync_points(points)
    it, rc = ctypes.c_int32(0), ctypes.c_double(0.0)
    r = _check(lib().eggsync_sync_lambda(_ptr(x), n, d, ctypes.c_float(eps), ctypes.c_double(lam), max_iters,
                                         dev, ctypes.byref(it), ctypes.byref(rc)), (OK, NOT_CONVERGED))
    return {"points": x, "iters": it.value, "rc": rc.value, "reached": r == OK}


class Context:
    """Device-resident phase API (eggsync_ctx_*), used by the multi-GPU driver and device-timed bench."""

    def __init__(self, n: int, d: int, eps: float, device: int = -1, stream=None):
        self.n, self.d, self.eps = n, d, eps
        h = ctypes.c_void_p()
        _check(lib().eggsync_ctx_create(n, d, ctypes.c_float(eps), device,
                                        ctypes.c_void_p(stream) if stream else None, ctypes.byref(h)))
        self.h = h

    def close(self):
        if self.h:
            lib().eggsync_ctx_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def load(self, points):
        on_dev = _is_torch_cuda(points)
        if not on_dev:
            points = _host_points(points)
        else:
            # order the context's stream after the work that produced the tensor
            import torch
            torch.cuda.ExternalStream(self.stream(), device=points.device).wait_stream(
                torch.cuda.current_stream(points.device))
        self._keep = points
        _check(lib().eggsync_ctx_load(self.h, _ptr(points), int(on_dev)))

    def build(self) -> int:
        nc = ctypes.c_int32(0)
        _check(lib().eggsync_ctx_build(self.h, ctypes.byref(nc)))
        return nc.value

    def update(self, lo: int = 0, hi: int | None = None):
        _check(lib().eggsync_ctx_update(self.h, lo, self.n if hi is None else hi))

    def second_term(self, lo: int = 0, hi: int | None = None):
        _check(lib().eggsync_ctx_second_term(self.h, lo, self.n if hi is None else hi))

    def flags(self):
        a, b = ctypes.c_int32(0), ctypes.c_int32(0)
        _check(lib().eggsync_ctx_flags(self.h, ctypes.byref(a), ctypes.byref(b)))
        return a.value, b.value

    def next_coords_ptr(self) -> int:
        return lib().eggsync_ctx_next_coords(self.h)

    def cur_coords_ptr(self) -> int:
        return lib().eggsync_ctx_cur_coords(self.h)

    def pack(self, lo: int, cnt: int, buf_ptr: int):
        _check(lib().eggsync_ctx_pack(self.h, lo, cnt, ctypes.c_void_p(buf_ptr)))

    def unpack(self, gathered_ptr: int, ranks: int, cnt: int):
        _check(lib().eggsync_ctx_unpack(self.h, ctypes.c_void_p(gathered_ptr), ranks, cnt))

    def pack_into(self, lo: int, cnt: int, tensor):
        """Next-state columns [lo, lo+cnt) into a CUDA tensor of shape (d, cnt)."""
        self.pack(lo, cnt, tensor.data_ptr())

    def unpack_from(self, tensor, ranks: int, cnt: int):
        """Gathered (ranks, d, cnt) CUDA tensor into the next-state buffer."""
        self.unpack(tensor.data_ptr(), ranks, cnt)

    # block-interleaved ownership (multi-GPU load balance)
    def update_owned(self, rank: int, ranks: int):
        _check(lib().eggsync_ctx_update_owned(self.h, rank, ranks))

    def owned_count(self, ranks: int) -> int:
        return int(lib().eggsync_ctx_owned_count(self.h, ranks))

    def pack_owned_into(self, rank: int, ranks: int, tensor):
        _check(lib().eggsync_ctx_pack_owned(self.h, rank, ranks, ctypes.c_void_p(tensor.data_ptr())))

    def set_own(self, n_own: int):
        """Sharded runs: the first n_own loaded points are this rank's own (criterion flags)."""
        _check(lib().eggsync_ctx_set_own(self.h, n_own))

    def plan_owned(self, rank: int, ranks: int):
        """Plan pass of the owned tiles; returns int64[6] statistics (see eggsync.h)."""
        out = np.zeros(6, np.int64)
        _check(lib().eggsync_ctx_plan_owned(self.h, rank, ranks, out.ctypes.data_as(ctypes.c_void_p)))
        return out

    def update_planned(self, rank: int, ranks: int, global_stats):
        """Update of the owned tiles with the kernel chosen from rank-reduced plan statistics."""
        g = np.ascontiguousarray(global_stats, dtype=np.int64)
        _check(lib().eggsync_ctx_update_planned(self.h, rank, ranks, g.ctypes.data_as(ctypes.c_void_p)))

    def unpack_owned_from(self, tensor, ranks: int):
        _check(lib().eggsync_ctx_unpack_owned(self.h, ctypes.c_void_p(tensor.data_ptr()), ranks))

    def advance(self):
        _check(lib().eggsync_ctx_advance(self.h))

    def labels(self, out=None):
        if out is None:
            out = np.empty(self.n, np.int32)
        _check(lib().eggsync_ctx_labels(self.h, _ptr(out), int(_is_torch_cuda(out))))
        return out

    def coords(self, out=None):
        if out is None:
            out = np.empty((self.n, self.d), np.float32)
        _check(lib().eggsync_ctx_coords(self.h, _ptr(out), int(_is_torch_cuda(out))))
        return out

    def run(self, max_iters: int = 10000):
        it = ctypes.c_int32(0)
        rc = lib().eggsync_ctx_run(self.h, max_iters, ctypes.byref(it))
        _check(rc, (OK, NOT_CONVERGED))
        return it.value, rc == OK

    def stream(self) -> int:
        return lib().eggsync_ctx_stream(self.h) or 0

    WORK_KEYS = ("cls", "acc", "scan", "node", "exact", "part", "nfull", "staged")

    def work(self, enable: int = -1):
        """Read the update's work counters (dict), then set counting on (1) / off (0) / unchanged (-1)."""
        out = np.zeros(8, np.int64)
        _check(lib().eggsync_ctx_work(self.h, enable, out.ctypes.data_as(ctypes.c_void_p)))
        return dict(zip(self.WORK_KEYS, out.tolist()))

    TC_KEYS = ("launches", "pairs", "pairs_padded", "flops", "ns")

    def tc_work(self, enable: int = -1):
        """Tensor-core update work / kernel time (dict), then set timing on (1) / off (0) / unchanged (-1)."""
        out = np.zeros(5, np.int64)
        _check(lib().eggsync_ctx_tc_work(self.h, enable, out.ctypes.data_as(ctypes.c_void_p)))
        return dict(zip(self.TC_KEYS, out.tolist()))

    def launches(self) -> int:
        return int(lib().eggsync_ctx_launches(self.h))

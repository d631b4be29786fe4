"""Python binding of libbar.so (include/bar.h): argument marshalling only.

Every step of the solve runs in the library's CUDA kernels; this module only converts
numpy arrays / torch tensors into pointers. It never falls back to a CPU path: if
``libbar.so`` is missing or fails to load, importing this module raises.

The C names are kept: ``bar_create_csr``, ``bar_solve``, ``bar_solve_ex``, ``bar_sweep``,
``bar_residual``, ``bar_matrix_get_info``, ``bar_set_tuning``, ``bar_destroy``,
``bar_last_error``. ``Matrix`` is a small RAII wrapper over them. The library reads no
environment variable: kernel / schedule overrides go through ``Matrix.set_tuning``.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("BAR_LIB") or os.path.join(_HERE, "libbar.so")  # BAR_LIB: A/B builds

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: run `python -c 'import __graft_entry__ as g; g.build()'` "
                      "(there is no CPU fallback)")
_lib = ctypes.CDLL(LIB_PATH)

MODE_ASYNC, MODE_SYNC_BLOCK, MODE_JACOBI = 0, 1, 2
MODES = {"async": MODE_ASYNC, "sync-block": MODE_SYNC_BLOCK, "jacobi": MODE_JACOBI}
STATUS = {0: "BAR_OK", 1: "BAR_ERR_INVALID_ARG", 2: "BAR_ERR_BAD_CSR", 3: "BAR_ERR_ZERO_DIAG",
          4: "BAR_ERR_NONFINITE", 5: "BAR_ERR_DIVERGED", 6: "BAR_ERR_CUDA", 7: "BAR_ERR_NCCL", 8: "BAR_ERR_OOM"}
MAX_ROWS_PER_BLOCK = 8192

# every symbol include/bar.h declares (tests check the export table against the header)
EXPORTS = ("bar_create_csr", "bar_solve", "bar_solve_ex", "bar_sweep", "bar_residual", "bar_matrix_get_info",
           "bar_set_tuning", "bar_destroy", "bar_last_error", "bar_create_csr_dist", "bar_nccl_unique_id",
           "bar_dist_ghosts", "bar_dist_localize", "bar_dist_plan", "bar_dist_create", "bar_dist_link_loopback",
           "bar_dist_solve", "bar_dist_solve_loopback", "bar_dist_sweep", "bar_dist_p2p_handles",
           "bar_dist_enable_p2p", "bar_dist_set_tuning", "bar_dist_destroy", "bar_build_id")


class SolveInfo(ctypes.Structure):
    _fields_ = [("iters", ctypes.c_int64), ("rel_res", ctypes.c_double), ("converged", ctypes.c_int32),
                ("cta_iters_min", ctypes.c_int64), ("cta_iters_max", ctypes.c_int64),
                ("model_bytes_per_iter", ctypes.c_double), ("kernel_launches", ctypes.c_int64),
                ("sweep_kernel_ms", ctypes.c_double), ("sweep_kernel_iters", ctypes.c_double)]

    def as_dict(self):
        return {f: getattr(self, f) for f, _ in self._fields_}


class SolveOpts(ctypes.Structure):
    _fields_ = [("tau", ctypes.c_double), ("fail_mask", ctypes.c_void_p), ("fail_start", ctypes.c_int64),
                ("fail_stop", ctypes.c_int64), ("res_history", ctypes.c_void_p),
                ("async_single_launch", ctypes.c_int32)]


class MatrixInfo(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int64), ("nnz", ctypes.c_int64), ("rows_per_block", ctypes.c_int32),
                ("num_subdomains", ctypes.c_int64), ("layout_entries", ctypes.c_int64),
                ("local_entries", ctypes.c_int64), ("model_bytes_per_iter", ctypes.c_double),
                ("device", ctypes.c_int32), ("last_sweep_kernel", ctypes.c_char_p), ("coded", ctypes.c_int32),
                ("layout_bytes_per_iter", ctypes.c_double)]

    def as_dict(self):
        d = {f: getattr(self, f) for f, _ in self._fields_}
        d["last_sweep_kernel"] = (d["last_sweep_kernel"] or b"").decode()
        return d


class Tuning(ctypes.Structure):
    """bar_tuning (include/bar.h): explicit per-handle kernel / schedule overrides; zero = defaults."""

    _fields_ = [(f, ctypes.c_int32) for f in (
        "kernel", "duo", "pipe", "coded", "async_order", "async_queue", "resident", "lead", "ghost_prefetch", "graph",
        "single_launch", "jacobi_rowwise", "grid_cap", "warps", "halo", "peer", "fronts",
        "stage_bx", "lazy_publish", "slab_prefetch", "overlap", "unroll_off", "fuse_residual", "gather_ahead")]

    KERNELS = {"auto": 0, "block": 1, "reg": 2, "reg_tma": 3, "pers": 4}
    ORDERS = {"auto": 0, "chunks": 1, "round_robin": 2, "fronts": 3}

    @classmethod
    def make(cls, **kw):
        """Tuning(kernel="block", duo=-1, async_order="round_robin", halo="allgather", ...)."""
        t = cls()
        for k, v in kw.items():
            if k == "kernel" and isinstance(v, str):
                v = cls.KERNELS[v]
            elif k == "async_order" and isinstance(v, str):
                v = cls.ORDERS[v]
            elif k == "async_queue" and isinstance(v, str):
                v = {"static": 0, "queue": 1}[v]
            elif k == "halo" and isinstance(v, str):
                v = {"sendrecv": 0, "allgather": 1}[v]
            elif isinstance(v, bool):
                v = 1 if v else -1
            if k not in dict(cls._fields_):
                raise KeyError(f"unknown bar_tuning field {k}")
            setattr(t, k, int(v))
        return t


_vp, _i64, _i32, _f64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_double
_lib.bar_set_tuning.restype = ctypes.c_int
_lib.bar_set_tuning.argtypes = [_vp, ctypes.POINTER(Tuning)]
_lib.bar_create_csr.restype = ctypes.c_int
_lib.bar_create_csr.argtypes = [_i64, _i64, _vp, _vp, _vp, _i32, ctypes.c_int, ctypes.POINTER(_vp)]
_lib.bar_solve.restype = ctypes.c_int
_lib.bar_solve.argtypes = [_vp, _vp, _vp, _vp, _i32, _i64, _f64, ctypes.c_int, _vp, ctypes.POINTER(SolveInfo)]
_lib.bar_solve_ex.restype = ctypes.c_int
_lib.bar_solve_ex.argtypes = [_vp, _vp, _vp, _vp, _i32, _i64, _f64, ctypes.c_int, _vp, ctypes.POINTER(SolveInfo),
                              ctypes.POINTER(SolveOpts)]
_lib.bar_sweep.restype = ctypes.c_int
_lib.bar_sweep.argtypes = [_vp, _vp, _vp, _i32, _i64, ctypes.c_int, _vp]
_lib.bar_residual.restype = ctypes.c_int
_lib.bar_residual.argtypes = [_vp, _vp, _vp, _vp, ctypes.POINTER(_f64), ctypes.POINTER(_f64)]
_lib.bar_matrix_get_info.restype = ctypes.c_int
_lib.bar_matrix_get_info.argtypes = [_vp, ctypes.POINTER(MatrixInfo)]
_lib.bar_destroy.restype = None
_lib.bar_destroy.argtypes = [_vp]
_lib.bar_last_error.restype = ctypes.c_char_p
_lib.bar_last_error.argtypes = []
_lib.bar_build_id.restype = ctypes.c_char_p
_lib.bar_build_id.argtypes = []


class BarError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status
        self.name = STATUS.get(status, str(status))


def _ptr(a):
    """Pointer of a contiguous numpy array or torch tensor (host or device); None -> NULL."""
    if a is None:
        return None
    if hasattr(a, "data_ptr"):
        if not a.is_contiguous():
            raise ValueError("tensor must be contiguous")
        return a.data_ptr()
    if isinstance(a, np.ndarray):
        if not a.flags["C_CONTIGUOUS"]:
            raise ValueError("array must be C-contiguous")
        return a.ctypes.data
    raise TypeError(f"unsupported array type {type(a)}")


def _check(st: int):
    if st != 0:
        raise BarError(st, bar_last_error())


def bar_last_error() -> str:
    return _lib.bar_last_error().decode()


def bar_build_id() -> str:
    return _lib.bar_build_id().decode()


def bar_create_csr(n, nnz, rowptr, col, val, rows_per_block, device=0):
    h = _vp()
    _check(_lib.bar_create_csr(n, nnz, _ptr(rowptr), _ptr(col), _ptr(val), rows_per_block, device, ctypes.byref(h)))
    return h


def bar_solve(A, b, x0, x, k, max_global_iters, tol, mode, cuda_stream=None, raise_on_error=True):
    info = SolveInfo()
    if isinstance(mode, str):
        mode = MODES[mode]
    st = _lib.bar_solve(A, _ptr(b), _ptr(x0), _ptr(x), k, max_global_iters, tol, mode, cuda_stream,
                        ctypes.byref(info))
    if raise_on_error:
        _check(st)
    return st, info


def bar_solve_ex(A, b, x0, x, k, max_global_iters, tol, mode, cuda_stream=None, raise_on_error=True, tau=1.0,
                 fail_mask=None, fail_start=0, fail_stop=-1, history=None, async_single_launch=-1):
    """bar_solve with the options struct (N1 failure injection, N3 tau-scaling, residual history)."""
    info = SolveInfo()
    if isinstance(mode, str):
        mode = MODES[mode]
    opts = SolveOpts(tau, None, fail_start, fail_stop, None, async_single_launch)
    keep = []
    if fail_mask is not None:
        m = fail_mask if hasattr(fail_mask, "data_ptr") else np.ascontiguousarray(fail_mask, dtype=np.uint8)
        keep.append(m)
        opts.fail_mask = _ptr(m)
    if history is not None:
        assert isinstance(history, np.ndarray) and history.dtype == np.float64 and len(history) >= max_global_iters + 1
        opts.res_history = history.ctypes.data
    st = _lib.bar_solve_ex(A, _ptr(b), _ptr(x0), _ptr(x), k, max_global_iters, tol, mode, cuda_stream,
                           ctypes.byref(info), ctypes.byref(opts))
    if raise_on_error:
        _check(st)
    return st, info


def bar_sweep(A, b, x, k, nsweeps, mode, cuda_stream=None):
    if isinstance(mode, str):
        mode = MODES[mode]
    _check(_lib.bar_sweep(A, _ptr(b), _ptr(x), k, nsweeps, mode, cuda_stream))


def bar_residual(A, b, x, cuda_stream=None):
    r, bn = _f64(), _f64()
    _check(_lib.bar_residual(A, _ptr(b), _ptr(x), cuda_stream, ctypes.byref(r), ctypes.byref(bn)))
    return r.value, bn.value


def bar_matrix_get_info(A):
    info = MatrixInfo()
    _check(_lib.bar_matrix_get_info(A, ctypes.byref(info)))
    return info


def bar_set_tuning(A, tuning=None):
    """tuning: a Tuning, a dict of its fields, or None (defaults)."""
    if isinstance(tuning, dict):
        tuning = Tuning.make(**tuning)
    _check(_lib.bar_set_tuning(A, ctypes.byref(tuning) if tuning is not None else None))


def bar_destroy(A):
    _lib.bar_destroy(A)


def _stream_handle(stream):
    if stream is None:
        try:
            import torch

            return torch.cuda.current_stream().cuda_stream
        except Exception:
            return None
    return getattr(stream, "cuda_stream", stream)


class Matrix:
    """A CSR matrix resident on a B200 in the library's layout (owns a bar_matrix handle)."""

    def __init__(self, rowptr, col, val, rows_per_block: int = 128, device: int = 0, n: int | None = None,
                 tuning=None):
        n = (len(rowptr) - 1) if n is None else n
        nnz = int(rowptr[-1]) if isinstance(rowptr, np.ndarray) else int(rowptr[-1].item())
        self.handle = bar_create_csr(n, nnz, rowptr, col, val, rows_per_block, device)
        self.n, self.nnz, self.R, self.device = n, nnz, rows_per_block, device
        if tuning:
            self.set_tuning(tuning)

    @classmethod
    def from_csr(cls, A, rows_per_block: int = 128, device: int = 0, tuning=None):
        """From a workloads.CSR (host numpy arrays)."""
        return cls(np.ascontiguousarray(A.rowptr, dtype=np.int32), np.ascontiguousarray(A.col, dtype=np.int32),
                   np.ascontiguousarray(A.val, dtype=np.float64), rows_per_block, device, n=A.n, tuning=tuning)

    def set_tuning(self, tuning=None, **kw):
        """bar_set_tuning: a Tuning, a dict, keyword fields, or nothing (defaults)."""
        bar_set_tuning(self.handle, tuning if tuning is not None or not kw else dict(kw))

    def info(self) -> dict:
        return bar_matrix_get_info(self.handle).as_dict()

    def solve(self, b, x0=None, x=None, k: int = 5, max_global_iters: int = 20000, tol: float = 1e-10,
              mode="async", stream=None, raise_on_error=True, tau=1.0, fail_mask=None, fail_start=0, fail_stop=-1,
              history=False, async_single_launch=-1):
        """Solve in place into ``x`` (allocated like ``b`` if None). Returns (x, info dict).

        Options (bar_solve_ex): ``tau`` (N3), ``fail_mask``/``fail_start``/``fail_stop`` (N1),
        ``history`` (info["history"] = rel_res per global iteration)."""
        if x is None:
            if hasattr(b, "data_ptr"):
                import torch

                x = torch.empty_like(b)
            else:
                x = np.empty_like(b)
        ext = tau != 1.0 or fail_mask is not None or history or async_single_launch != -1
        hist = np.full(max_global_iters + 1, np.nan) if history else None
        if ext:
            st, info = bar_solve_ex(self.handle, b, x0, x, k, max_global_iters, tol, mode, _stream_handle(stream),
                                    raise_on_error, tau, fail_mask, fail_start, fail_stop, hist, async_single_launch)
        else:
            st, info = bar_solve(self.handle, b, x0, x, k, max_global_iters, tol, mode, _stream_handle(stream),
                                 raise_on_error)
        d = info.as_dict()
        d["status"] = STATUS.get(st, st)
        if hist is not None:
            d["history"] = hist[: d["iters"] + 1]
        return x, d

    def sweep(self, b, x, k: int = 5, nsweeps: int = 1, mode="async", stream=None):
        """Enqueue exactly ``nsweeps`` global iterations (no convergence control, no sync)."""
        bar_sweep(self.handle, b, x, k, nsweeps, mode, _stream_handle(stream))

    def residual(self, b, x, stream=None):
        return bar_residual(self.handle, b, x, _stream_handle(stream))

    def close(self):
        if getattr(self, "handle", None):
            bar_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

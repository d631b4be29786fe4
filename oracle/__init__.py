"""TEST INFRASTRUCTURE ONLY — the CPU oracle for block-asynchronous relaxation.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py`` (its ``cpu_baseline``
leg and ``--impl reference``) may import this package. The CUDA product path
(``paper_conf_ipps_anzttdh12_b200``) never imports it and shares no code with it.

Thin ctypes wrapper around ``oracle/oracle.c`` (single-threaded C, fp64,
``-ffp-contract=off``); see that file's header for the paper passage each function
follows (O1 Jacobi eq. 2; O2 sync-block-(k) Alg. 1 P:149-163 / eq. 4
P:177-209; O3 Gauss-Seidel P:91/P:139; O4 residual P:523; O5 stopping rule).

Parity status: O1-O5 are pinned by tests/test_oracle.py.
"Parity unpinned": the exact asynchronous iterate sequence (nondeterministic by
design, eq. 3) — async is validated by outcome, never iterate-by-iterate.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None

JACOBI, BLOCK_JACOBI, GAUSS_SEIDEL = 0, 1, 2
OK, ERR, DIVERGED = 0, 1, 2


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        from tools.build import build_oracle

        build_oracle()
    lib = ctypes.CDLL(_LIB_PATH)
    i64, i32 = ctypes.c_int64, ctypes.c_int32
    i32p, f64p = ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_double)
    lib.oracle_residual_norm.restype = ctypes.c_double
    lib.oracle_residual_norm.argtypes = [i64, i32p, i32p, f64p, f64p, f64p]
    lib.oracle_norm2.restype = ctypes.c_double
    lib.oracle_norm2.argtypes = [i64, f64p]
    lib.oracle_jacobi_rows.restype = ctypes.c_int
    lib.oracle_jacobi_rows.argtypes = [i64, i64, i32p, i32p, f64p, f64p, f64p, f64p]
    lib.oracle_jacobi_step.restype = ctypes.c_int
    lib.oracle_jacobi_step.argtypes = [i64, i32p, i32p, f64p, f64p, f64p, f64p]
    lib.oracle_block_jacobi_subdomain.restype = ctypes.c_int
    lib.oracle_block_jacobi_subdomain.argtypes = [i64, i64, i32p, i32p, f64p, f64p, f64p, i32, f64p, f64p]
    lib.oracle_block_jacobi_step.restype = ctypes.c_int
    lib.oracle_block_jacobi_step.argtypes = [i64, i32p, i32p, f64p, f64p, i64, i32, f64p, f64p]
    lib.oracle_gauss_seidel_step.restype = ctypes.c_int
    lib.oracle_gauss_seidel_step.argtypes = [i64, i32p, i32p, f64p, f64p, f64p]
    lib.oracle_solve.restype = ctypes.c_int
    lib.oracle_solve.argtypes = [i32, i64, i32p, i32p, f64p, f64p, f64p, f64p, i64, i32, i64, ctypes.c_double,
                                 ctypes.POINTER(i64), f64p, ctypes.POINTER(i32), f64p]
    u8p = ctypes.POINTER(ctypes.c_uint8)
    lib.oracle_solve_ex.restype = ctypes.c_int
    lib.oracle_solve_ex.argtypes = lib.oracle_solve.argtypes + [ctypes.c_double, u8p, i64, i64]
    lib.oracle_jacobi_step_ex.restype = ctypes.c_int
    lib.oracle_jacobi_step_ex.argtypes = [i64, i32p, i32p, f64p, f64p, f64p, f64p, ctypes.c_double, u8p]
    lib.oracle_block_jacobi_step_ex.restype = ctypes.c_int
    lib.oracle_block_jacobi_step_ex.argtypes = [i64, i32p, i32p, f64p, f64p, i64, i32, f64p, f64p, ctypes.c_double,
                                                u8p]
    _lib = lib
    return lib


def _i32(a):
    a = np.ascontiguousarray(a, dtype=np.int32)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_int32))


def _f64(a):
    a = np.ascontiguousarray(a, dtype=np.float64)
    return a, a.ctypes.data_as(ctypes.POINTER(ctypes.c_double))


def residual_norm(A, b, x) -> float:
    """O4: ||b - A x||_2 (A is a workloads.CSR over all n rows)."""
    lib = _load()
    rp, prp = _i32(A.rowptr)
    c, pc = _i32(A.col)
    v, pv = _f64(A.val)
    bb, pb = _f64(b)
    xx, px = _f64(x)
    return lib.oracle_residual_norm(len(rp) - 1, prp, pc, pv, pb, px)


def norm2(v) -> float:
    vv, pv = _f64(v)
    return _load().oracle_norm2(len(vv), pv)


def rel_res(A, b, x) -> float:
    return residual_norm(A, b, x) / norm2(b)


def jacobi_step(A, b, x_old) -> np.ndarray:
    """O1: one Jacobi iteration (eq. 2)."""
    lib = _load()
    rp, prp = _i32(A.rowptr)
    c, pc = _i32(A.col)
    v, pv = _f64(A.val)
    bb, pb = _f64(b)
    xo, pxo = _f64(x_old)
    out = np.empty(len(rp) - 1)
    if lib.oracle_jacobi_step(len(rp) - 1, prp, pc, pv, pb, pxo, out.ctypes.data_as(ctypes.POINTER(ctypes.c_double))):
        raise ValueError("zero diagonal")
    return out


def jacobi_rows(A_rows, b_rows, x_old) -> np.ndarray:
    """O1 on the row block A_rows (a workloads.CSR row range, global columns) given the full x_old."""
    lib = _load()
    rp, prp = _i32(A_rows.rowptr)
    c, pc = _i32(A_rows.col)
    v, pv = _f64(A_rows.val)
    bb, pb = _f64(b_rows)
    xo, pxo = _f64(x_old)
    out = np.empty(len(rp) - 1)
    if lib.oracle_jacobi_rows(A_rows.row_lo, len(rp) - 1, prp, pc, pv, pb, pxo,
                              out.ctypes.data_as(ctypes.POINTER(ctypes.c_double))):
        raise ValueError("zero diagonal")
    return out


def block_jacobi_step(A, b, x_old, R: int, k: int) -> np.ndarray:
    """O2: one global iteration of sync-block-(k) with subdomains of R rows (Alg. 1)."""
    lib = _load()
    rp, prp = _i32(A.rowptr)
    c, pc = _i32(A.col)
    v, pv = _f64(A.val)
    bb, pb = _f64(b)
    xo, pxo = _f64(x_old)
    out = np.empty(len(rp) - 1)
    rc = lib.oracle_block_jacobi_step(len(rp) - 1, prp, pc, pv, pb, R, k, pxo,
                                      out.ctypes.data_as(ctypes.POINTER(ctypes.c_double)))
    if rc:
        raise ValueError(f"oracle_block_jacobi_step failed ({rc})")
    return out


def block_jacobi_subdomain(A_rows, b_rows, x_old, k: int) -> np.ndarray:
    """O2 for the single subdomain J = [A_rows.row_lo, A_rows.row_hi) given the full x^m."""
    lib = _load()
    rp, prp = _i32(A_rows.rowptr)
    c, pc = _i32(A_rows.col)
    v, pv = _f64(A_rows.val)
    bb, pb = _f64(b_rows)
    xo, pxo = _f64(x_old)
    nl = len(rp) - 1
    out = np.empty(nl)
    work = np.empty(2 * max(nl, 1))
    rc = lib.oracle_block_jacobi_subdomain(A_rows.row_lo, A_rows.row_hi, prp, pc, pv, pb, pxo, k,
                                           out.ctypes.data_as(ctypes.POINTER(ctypes.c_double)),
                                           work.ctypes.data_as(ctypes.POINTER(ctypes.c_double)))
    if rc:
        raise ValueError("zero diagonal")
    return out


def gauss_seidel_step(A, b, x) -> np.ndarray:
    """O3: one forward Gauss-Seidel sweep; returns a new array."""
    lib = _load()
    rp, prp = _i32(A.rowptr)
    c, pc = _i32(A.col)
    v, pv = _f64(A.val)
    bb, pb = _f64(b)
    out = np.array(x, dtype=np.float64, copy=True)
    if lib.oracle_gauss_seidel_step(len(rp) - 1, prp, pc, pv, pb, out.ctypes.data_as(ctypes.POINTER(ctypes.c_double))):
        raise ValueError("zero diagonal")
    return out


@dataclass
class SolveResult:
    x: np.ndarray
    iters: int
    rel_res: float
    converged: bool
    status: int
    history: np.ndarray


def solve(A, b, x0=None, method: int = BLOCK_JACOBI, R: int = 128, k: int = 5,
          max_iters: int = 20000, tol: float = 1e-10, tau: float = 1.0, frozen=None,
          fail_start: int = 0, fail_stop: int = -1) -> SolveResult:
    """O5: iterate until rel_res(x^m) <= tol (first such m) or max_iters.

    N3: ``tau`` scales every update (B = I - tau D^-1 A). N1: components with
    ``frozen[i]`` do not update in global iterations fail_start <= m < fail_stop."""
    lib = _load()
    n = len(A.rowptr) - 1
    rp, prp = _i32(A.rowptr)
    c, pc = _i32(A.col)
    v, pv = _f64(A.val)
    bb, pb = _f64(b)
    if x0 is None:
        x0 = np.zeros(n)
    xx0, px0 = _f64(x0)
    out = np.empty(n)
    hist = np.full(max_iters + 1, np.nan)
    iters = ctypes.c_int64()
    rel = ctypes.c_double()
    conv = ctypes.c_int32()
    fz = None
    pfz = None
    if frozen is not None:
        fz = np.ascontiguousarray(frozen, dtype=np.uint8)
        pfz = fz.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8))
    st = lib.oracle_solve_ex(method, n, prp, pc, pv, pb, px0, out.ctypes.data_as(ctypes.POINTER(ctypes.c_double)),
                             R, k, max_iters, tol, ctypes.byref(iters), ctypes.byref(rel), ctypes.byref(conv),
                             hist.ctypes.data_as(ctypes.POINTER(ctypes.c_double)), tau, pfz, fail_start, fail_stop)
    if st == ERR:
        raise ValueError("oracle_solve failed")
    return SolveResult(out, iters.value, rel.value, bool(conv.value), st, hist[: iters.value + 1])


def step_ex(A, b, x_old, method: int = BLOCK_JACOBI, R: int = 128, k: int = 5, tau: float = 1.0, frozen=None):
    """One global iteration of O1/O2 with the N1/N3 options."""
    lib = _load()
    n = len(A.rowptr) - 1
    rp, prp = _i32(A.rowptr)
    c, pc = _i32(A.col)
    v, pv = _f64(A.val)
    bb, pb = _f64(b)
    xo, pxo = _f64(x_old)
    out = np.empty(n)
    po = out.ctypes.data_as(ctypes.POINTER(ctypes.c_double))
    pfz = None
    if frozen is not None:
        fz = np.ascontiguousarray(frozen, dtype=np.uint8)
        pfz = fz.ctypes.data_as(ctypes.POINTER(ctypes.c_uint8))
    if method == JACOBI:
        rc = lib.oracle_jacobi_step_ex(n, prp, pc, pv, pb, pxo, po, tau, pfz)
    else:
        rc = lib.oracle_block_jacobi_step_ex(n, prp, pc, pv, pb, R, k, pxo, po, tau, pfz)
    if rc:
        raise ValueError("step failed")
    return out

"""Seeded / deterministic synthetic inputs shared by the oracle side and the CUDA side.

This module holds none of the method's arithmetic (no splitting, no sweep, no
residual): it only builds the paper's test matrices and right-hand sides.

* ``trefethen(n)`` — Trefethen_2000 / Trefethen_20000 exactly (Table 1,
  P:129): primes on the diagonal, ones at |i-j| = 2^t.
* ``stencil9_2d(m, diag)`` — fv1/fv2/fv3 pattern (9-point, m x m grid, Table 1
  P:129), configs C2 and C4.
* ``stencil7_3d(m, diag)`` — 3D 7-point (config C5, BASELINE.json configs[4]).
* ``random_dd(n, ...)`` — seeded random sparse diagonally dominant matrices for
  property tests (numpy ``default_rng(seed)``).
* ``dyadic_stencil9_2d(m, p)`` — diagonal 2^p, off-diagonal -1: every Jacobi-type
  iterate with integer b is an exact dyadic rational.

All generators return CSR as numpy arrays ``(rowptr int32, col int32, val float64)``
with strictly ascending columns and the diagonal present. Row ranges
``[row_lo, row_hi)`` with global column ids are supported for multi-GPU ranks and
for sampled parity checks at full size.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libworkloads.so")
_lib = None

# Diagonals chosen in SURVEY.md §8(c) P3 / §8(d): fv1's rho(B)=0.8541 for the 2D
# 9-point stencil, and 6/0.8541 for the 3D 7-point stencil.
FV1_DIAG = 9.3595
S7_DIAG = 7.0249


def _load():
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(_LIB_PATH):
        from tools.build import build_workloads  # noqa: WPS433 (CPU-only gcc build)
        build_workloads()
    lib = ctypes.CDLL(_LIB_PATH)
    i64, i32p, f64p = ctypes.c_int64, ctypes.POINTER(ctypes.c_int32), ctypes.POINTER(ctypes.c_double)
    lib.gen_trefethen_nnz.restype = i64
    lib.gen_trefethen_nnz.argtypes = [i64, i64, i64]
    lib.gen_trefethen.restype = ctypes.c_int
    lib.gen_trefethen.argtypes = [i64, i64, i64, i32p, i32p, f64p]
    lib.gen_stencil9_2d_nnz.restype = i64
    lib.gen_stencil9_2d_nnz.argtypes = [i64, i64, i64]
    lib.gen_stencil9_2d.restype = ctypes.c_int
    lib.gen_stencil9_2d.argtypes = [i64, ctypes.c_double, ctypes.c_double, i64, i64, i32p, i32p, f64p]
    lib.gen_stencil7_3d_nnz.restype = i64
    lib.gen_stencil7_3d_nnz.argtypes = [i64, i64, i64]
    lib.gen_stencil7_3d.restype = ctypes.c_int
    lib.gen_stencil7_3d.argtypes = [i64, ctypes.c_double, ctypes.c_double, i64, i64, i32p, i32p, f64p]
    lib.gen_fill.restype = None
    lib.gen_fill.argtypes = [f64p, i64, ctypes.c_double]
    _lib = lib
    return lib


def _p(a, t):
    return a.ctypes.data_as(ctypes.POINTER(t))


@dataclass
class CSR:
    """Host CSR matrix (rows [row_lo, row_hi) of an n x n matrix, global column ids)."""

    n: int
    rowptr: np.ndarray
    col: np.ndarray
    val: np.ndarray
    row_lo: int = 0
    row_hi: int = -1
    name: str = ""

    def __post_init__(self):
        if self.row_hi < 0:
            self.row_hi = self.n

    @property
    def nnz(self) -> int:
        return int(self.rowptr[-1])

    def to_scipy(self):
        import scipy.sparse as sp

        return sp.csr_matrix((self.val, self.col, self.rowptr), shape=(self.row_hi - self.row_lo, self.n))

    def to_dense(self) -> np.ndarray:
        d = np.zeros((self.row_hi - self.row_lo, self.n))
        for r in range(self.row_hi - self.row_lo):
            s, e = self.rowptr[r], self.rowptr[r + 1]
            d[r, self.col[s:e]] = self.val[s:e]
        return d


def _gen(nnz_fn, fill_fn, n, row_lo, row_hi, *args, name=""):
    if row_hi is None:
        row_hi = n
    nnz = nnz_fn(*args[:1], row_lo, row_hi) if nnz_fn is not None else None
    if nnz < 0:
        raise ValueError("bad generator arguments")
    rowptr = np.empty(row_hi - row_lo + 1, dtype=np.int32)
    col = np.empty(max(nnz, 1), dtype=np.int32)[:nnz]
    val = np.empty(max(nnz, 1), dtype=np.float64)[:nnz]
    rc = fill_fn(*args, row_lo, row_hi, _p(rowptr, ctypes.c_int32), _p(col, ctypes.c_int32), _p(val, ctypes.c_double))
    if rc != 0:
        raise ValueError("generator failed")
    return CSR(n, rowptr, col, val, row_lo, row_hi, name)


def trefethen(n: int, row_lo: int = 0, row_hi: int | None = None) -> CSR:
    lib = _load()
    return _gen(lib.gen_trefethen_nnz, lib.gen_trefethen, n, row_lo, row_hi, n, name=f"Trefethen_{n}")


def stencil9_2d(m: int, diag: float = FV1_DIAG, off: float = -1.0, row_lo: int = 0, row_hi: int | None = None) -> CSR:
    lib = _load()
    n = m * m
    if row_hi is None:
        row_hi = n
    nnz = lib.gen_stencil9_2d_nnz(m, row_lo, row_hi)
    if nnz < 0:
        raise ValueError("bad generator arguments")
    rowptr = np.empty(row_hi - row_lo + 1, dtype=np.int32)
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=np.float64)
    rc = lib.gen_stencil9_2d(m, diag, off, row_lo, row_hi, _p(rowptr, ctypes.c_int32), _p(col, ctypes.c_int32),
                             _p(val, ctypes.c_double))
    if rc != 0:
        raise ValueError("generator failed")
    return CSR(n, rowptr, col, val, row_lo, row_hi, f"stencil9_2d_m{m}")


def stencil7_3d(m: int, diag: float = S7_DIAG, off: float = -1.0, row_lo: int = 0, row_hi: int | None = None) -> CSR:
    lib = _load()
    n = m * m * m
    if row_hi is None:
        row_hi = n
    nnz = lib.gen_stencil7_3d_nnz(m, row_lo, row_hi)
    if nnz < 0:
        raise ValueError("bad generator arguments")
    rowptr = np.empty(row_hi - row_lo + 1, dtype=np.int32)
    col = np.empty(nnz, dtype=np.int32)
    val = np.empty(nnz, dtype=np.float64)
    rc = lib.gen_stencil7_3d(m, diag, off, row_lo, row_hi, _p(rowptr, ctypes.c_int32), _p(col, ctypes.c_int32),
                             _p(val, ctypes.c_double))
    if rc != 0:
        raise ValueError("generator failed")
    return CSR(n, rowptr, col, val, row_lo, row_hi, f"stencil7_3d_m{m}")


def ones(n: int) -> np.ndarray:
    """b = 1 (SURVEY.md §8(c) reading 1), filled natively for the 128M-row config."""
    out = np.empty(n, dtype=np.float64)
    _load().gen_fill(_p(out, ctypes.c_double), n, 1.0)
    return out


def random_dd(n: int, nnz_per_row: int = 5, seed: int = 0, dominance: float = 1.5,
              symmetric_pattern: bool = False, negative: bool = False) -> CSR:
    """Seeded random sparse matrix with rho(|D^-1(L+U)|) <= 1/dominance < 1.

    Off-diagonals uniform in [-1, 1] (or [-1, 0] if ``negative``); the diagonal is
    ``dominance * sum_j |a_ij|`` (at least 1), so |B| has row sums <= 1/dominance.
    """
    rng = np.random.default_rng(seed)
    rows = []
    for i in range(n):
        k = min(n - 1, int(rng.integers(0, 2 * nnz_per_row)))
        others = rng.choice(np.delete(np.arange(n), i), size=k, replace=False) if k > 0 else np.array([], dtype=np.int64)
        vals = rng.uniform(-1.0, 0.0 if negative else 1.0, size=k)
        rows.append((others, vals))
    if symmetric_pattern:
        # mirror entries so the pattern (and values) are symmetric
        dense = {}
        for i, (c, v) in enumerate(rows):
            for j, a in zip(c, v):
                dense[(i, int(j))] = a
                dense[(int(j), i)] = a
        rows = [[[], []] for _ in range(n)]
        for (i, j), a in dense.items():
            rows[i][0].append(j)
            rows[i][1].append(a)
        rows = [(np.array(c, dtype=np.int64), np.array(v)) for c, v in rows]
    rowptr = [0]
    cols, vals = [], []
    for i, (c, v) in enumerate(rows):
        d = max(1.0, dominance * float(np.abs(v).sum()))
        cc = np.concatenate([c, [i]]).astype(np.int64)
        vv = np.concatenate([v, [d]])
        order = np.argsort(cc, kind="stable")
        cols.append(cc[order])
        vals.append(vv[order])
        rowptr.append(rowptr[-1] + len(cc))
    return CSR(n, np.array(rowptr, dtype=np.int32), np.concatenate(cols).astype(np.int32),
               np.concatenate(vals).astype(np.float64), 0, n, f"random_dd_n{n}_s{seed}")


def dyadic_stencil9_2d(m: int, p: int = 4) -> CSR:
    """9-point stencil with diagonal 2^p and off-diagonals -1."""
    return stencil9_2d(m, float(2 ** p), -1.0)

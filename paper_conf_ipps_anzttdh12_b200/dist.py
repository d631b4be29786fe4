"""Multi-GPU row-partitioned solve: Python side of include/bar.h's multi-GPU calls.

Marshalling only. Planning (ghost lists, the exchange plan, local numbering), the NCCL
communicator, the peer-memory mapping, the halo exchange, the sweeps and the residual all run
in libbar.so. Paper: §3.4, SURVEY.md §8(e).

* ``partition`` — contiguous, subdomain-aligned row ranges (rank p owns subdomains
  [p q / P, (p+1) q / P)).
* ``ghosts``, ``localize``, ``make_plan``, ``ghost_sources`` — the host-only planning calls
  (bar_dist_ghosts / bar_dist_localize / bar_dist_plan); no GPU needed.
* ``DistMatrix`` — one rank's share through ``bar_create_csr_dist`` (§8(b)): the library
  plans everything over NCCL; the caller only passes the 128-byte NCCL id around.
* ``PeerRank`` — one rank of separate processes WITHOUT NCCL (explicit plan, peer memory
  through CUDA IPC): the async mode only; used to run the collective-free peer-memory path
  with several processes on one GPU.
* ``LoopbackGroup`` — several ranks in one process on one GPU (device copies as the exchange).
"""
from __future__ import annotations

import ctypes

import numpy as np

from .bar import (MODES, STATUS, BarError, SolveInfo, Tuning, _check, _lib, _ptr, _stream_handle, bar_matrix_get_info,
                  bar_residual, bar_set_tuning, bar_solve, bar_sweep)

_vp, _i64, _i32, _f64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_double
_lib.bar_dist_ghosts.restype = ctypes.c_int
_lib.bar_dist_ghosts.argtypes = [_i64, _i64, _i64, _vp, _vp, ctypes.POINTER(_i64), ctypes.POINTER(_i64), _vp]
_lib.bar_dist_localize.restype = ctypes.c_int
_lib.bar_dist_localize.argtypes = [_i64, _i64, _i64, _vp, _vp, _i64, _i64, _vp, _vp]
_lib.bar_dist_plan.restype = ctypes.c_int
_lib.bar_dist_plan.argtypes = [ctypes.c_int, ctypes.c_int, _vp, _vp, _vp, _vp, _vp, _vp, _vp]
_lib.bar_nccl_unique_id.restype = ctypes.c_int
_lib.bar_nccl_unique_id.argtypes = [_vp]
_lib.bar_create_csr_dist.restype = ctypes.c_int
_lib.bar_create_csr_dist.argtypes = [_i64, _i64, _i64, _i64, _vp, _vp, _vp, _i32, ctypes.c_int, _vp, ctypes.c_int,
                                     ctypes.c_int, ctypes.POINTER(_vp)]
_lib.bar_dist_create.restype = ctypes.c_int
_lib.bar_dist_create.argtypes = [_i64, _i64, _i64, _i64, _vp, _vp, _vp, _i64, _i64, ctypes.c_int, ctypes.c_int, _vp,
                                 _vp, _vp, _i32, ctypes.c_int, _vp, ctypes.POINTER(_vp)]
_lib.bar_dist_link_loopback.restype = ctypes.c_int
_lib.bar_dist_link_loopback.argtypes = [ctypes.POINTER(_vp), ctypes.c_int]
_lib.bar_dist_solve.restype = ctypes.c_int
_lib.bar_dist_solve.argtypes = [_vp, _vp, _vp, _vp, _i32, _i64, _f64, ctypes.c_int, _vp, ctypes.POINTER(SolveInfo)]
_lib.bar_dist_solve_loopback.restype = ctypes.c_int
_lib.bar_dist_solve_loopback.argtypes = [ctypes.POINTER(_vp), ctypes.c_int, ctypes.POINTER(_vp), ctypes.POINTER(_vp),
                                         ctypes.POINTER(_vp), _i32, _i64, _f64, ctypes.c_int, _vp,
                                         ctypes.POINTER(SolveInfo)]
_lib.bar_dist_p2p_handles.restype = ctypes.c_int
_lib.bar_dist_p2p_handles.argtypes = [_vp, _vp, ctypes.POINTER(_i64)]
_lib.bar_dist_enable_p2p.restype = ctypes.c_int
_lib.bar_dist_enable_p2p.argtypes = [_vp, _vp, _vp, _vp]
_lib.bar_dist_sweep.restype = ctypes.c_int
_lib.bar_dist_sweep.argtypes = [_vp, _i32, _i64, ctypes.c_int, _vp]
_lib.bar_dist_set_tuning.restype = ctypes.c_int
_lib.bar_dist_set_tuning.argtypes = [_vp, ctypes.POINTER(Tuning)]
_lib.bar_dist_destroy.restype = None
_lib.bar_dist_destroy.argtypes = [_vp]


def _mode(m):
    return MODES[m] if isinstance(m, str) else m


def _info(st, info):
    d = info.as_dict()
    d["status"] = STATUS.get(st, st)
    return d


def _tuning(t):
    if t is None:
        return None
    return ctypes.byref(Tuning.make(**t) if isinstance(t, dict) else t)


def nccl_unique_id() -> bytes:
    """bar_nccl_unique_id: the 128-byte id rank 0 hands to every rank."""
    buf = ctypes.create_string_buffer(128)
    _check(_lib.bar_nccl_unique_id(buf))
    return buf.raw


def ghosts(A_rows):
    """Sorted ghost columns of a row block (workloads.CSR with row_lo/row_hi): (below, above)."""
    rp = np.ascontiguousarray(A_rows.rowptr, dtype=np.int32)
    col = np.ascontiguousarray(A_rows.col, dtype=np.int32)
    nlo, nhi = _i64(), _i64()
    _check(_lib.bar_dist_ghosts(A_rows.row_lo, A_rows.row_hi, len(col), _ptr(rp), _ptr(col), ctypes.byref(nlo),
                                ctypes.byref(nhi), None))
    g = np.empty(nlo.value + nhi.value, dtype=np.int32)
    _check(_lib.bar_dist_ghosts(A_rows.row_lo, A_rows.row_hi, len(col), _ptr(rp), _ptr(col), ctypes.byref(nlo),
                                ctypes.byref(nhi), _ptr(g)))
    return g[:nlo.value], g[nlo.value:]


def localize(A_rows, lo, hi):
    """Order-preserving local column numbering (ghosts below negative, above after the rows)."""
    rp = np.ascontiguousarray(A_rows.rowptr, dtype=np.int32)
    col = np.ascontiguousarray(A_rows.col, dtype=np.int32)
    g = np.ascontiguousarray(np.concatenate([lo, hi]), dtype=np.int32)
    out = np.empty_like(col)
    _check(_lib.bar_dist_localize(A_rows.row_lo, A_rows.row_hi, len(col), _ptr(rp), _ptr(col), len(lo), len(hi),
                                  _ptr(g), _ptr(out)))
    return out


def partition(n: int, R: int, nranks: int):
    """Contiguous row ranges aligned to subdomains: rank p owns subdomains [p q / P, (p+1) q / P)."""
    q = (n + R - 1) // R
    bounds = [min(n, (p * q // nranks) * R) for p in range(nranks + 1)]
    bounds[-1] = n
    return [(bounds[p], bounds[p + 1]) for p in range(nranks)]


def plan(rank: int, ranges, ghost_lists):
    """bar_dist_plan: (recv_counts, send_counts, send_idx, ghost_src_idx) of `rank` from every
    rank's row range and sorted ghost list."""
    P = len(ranges)
    rr = np.ascontiguousarray(np.asarray(ranges, dtype=np.int64).reshape(-1))
    gc = np.array([len(g) for g in ghost_lists], dtype=np.int64)
    ga = np.ascontiguousarray(np.concatenate([np.asarray(g, dtype=np.int32) for g in ghost_lists])
                              if gc.sum() else np.zeros(1, np.int32), dtype=np.int32)
    rc = np.zeros(P, dtype=np.int64)
    sc = np.zeros(P, dtype=np.int64)
    gs = np.zeros(max(1, int(gc[rank])), dtype=np.int32)
    _check(_lib.bar_dist_plan(P, rank, _ptr(rr), _ptr(gc), _ptr(ga), _ptr(rc), _ptr(sc), None, _ptr(gs)))
    si = np.zeros(max(1, int(sc.sum())), dtype=np.int32)
    _check(_lib.bar_dist_plan(P, rank, _ptr(rr), _ptr(gc), _ptr(ga), _ptr(rc), _ptr(sc), _ptr(si), None))
    return rc, sc, si[:int(sc.sum())], gs[:int(gc[rank])]


def make_plan(rank: int, ranges, ghost_lists):
    """recv_counts, send_counts, send_idx of `rank` (bar_dist_plan)."""
    rc, sc, si, _ = plan(rank, ranges, ghost_lists)
    return rc, sc, si


def ghost_sources(ranges, ghost_cols):
    """Owner-local row of every ghost column (ghost order), for bar_dist_enable_p2p."""
    g = np.asarray(ghost_cols, dtype=np.int64)
    if len(g) == 0:
        return np.zeros(0, dtype=np.int32)
    starts = np.array([r[0] for r in ranges])
    ends = np.array([r[1] for r in ranges])
    o = np.searchsorted(ends, g, side="right")
    return np.ascontiguousarray(g - starts[o], dtype=np.int32)


def _create(n_global, A_rows, R, device, nranks, rank, recv_counts, send_counts, send_idx, lo, hi, nccl_id):
    col_local = localize(A_rows, lo, hi)
    rp = np.ascontiguousarray(A_rows.rowptr, dtype=np.int32)
    val = np.ascontiguousarray(A_rows.val, dtype=np.float64)
    h = _vp()
    idbuf = ctypes.create_string_buffer(bytes(nccl_id), 128) if nccl_id is not None else None
    _check(_lib.bar_dist_create(n_global, A_rows.row_lo, A_rows.row_hi, len(col_local), _ptr(rp), _ptr(col_local),
                                _ptr(val), len(lo), len(hi), nranks, rank, _ptr(recv_counts), _ptr(send_counts),
                                _ptr(send_idx), R, device, idbuf, ctypes.byref(h)))
    return h


class DistMatrix:
    """One rank's share through bar_create_csr_dist (§8(b)): a bar_matrix handle whose bar_solve /
    bar_residual are collective over the NCCL group. Everything but the 128-byte NCCL id (rank 0's
    ``nccl_unique_id()``, handed to every rank by any means) happens inside libbar."""

    def __init__(self, A_rows, n_global: int, rows_per_block: int, device: int, nccl_id: bytes, rank: int,
                 nranks: int, tuning=None):
        rp = np.ascontiguousarray(A_rows.rowptr, dtype=np.int32)
        col = np.ascontiguousarray(A_rows.col, dtype=np.int32)
        val = np.ascontiguousarray(A_rows.val, dtype=np.float64)
        idbuf = ctypes.create_string_buffer(bytes(nccl_id), 128)
        h = _vp()
        _check(_lib.bar_create_csr_dist(n_global, A_rows.row_lo, A_rows.row_hi, len(col), _ptr(rp), _ptr(col),
                                        _ptr(val), rows_per_block, device, idbuf, rank, nranks, ctypes.byref(h)))
        self.handle = h
        self.rank, self.nranks, self.n_local = rank, nranks, A_rows.row_hi - A_rows.row_lo
        self.row_lo, self.row_hi = A_rows.row_lo, A_rows.row_hi
        if tuning:
            self.set_tuning(tuning)

    @classmethod
    def from_process_group(cls, A_rows, n_global, rows_per_block, device, group=None, tuning=None):
        """Rank 0 creates the NCCL id; torch.distributed only broadcasts those 128 bytes."""
        import torch.distributed as dist

        P, r = dist.get_world_size(group), dist.get_rank(group)
        nid = [nccl_unique_id() if r == 0 else None]
        dist.broadcast_object_list(nid, src=0, group=group)
        return cls(A_rows, n_global, rows_per_block, device, nid[0], r, P, tuning)

    def set_tuning(self, tuning=None, **kw):
        bar_set_tuning(self.handle, tuning if tuning is not None or not kw else dict(kw))

    def info(self) -> dict:
        return bar_matrix_get_info(self.handle).as_dict()

    def solve(self, b, x0=None, x=None, k=5, max_global_iters=20000, tol=1e-10, mode="async", stream=None,
              raise_on_error=True):
        if x is None:
            import torch

            x = torch.empty_like(b) if hasattr(b, "data_ptr") else np.empty_like(b)
        st, info = bar_solve(self.handle, b, x0, x, k, max_global_iters, tol, mode, _stream_handle(stream),
                             raise_on_error)
        return x, _info(st, info)

    def residual(self, b, x, stream=None):
        return bar_residual(self.handle, b, x, _stream_handle(stream))

    def sweep(self, b, x, k=5, nsweeps=1, mode="async", stream=None):
        """Enqueue nsweeps local block-sweep launches on this rank's rows (no exchange): kernel timing."""
        bar_sweep(self.handle, b, x, k, nsweeps, mode, _stream_handle(stream))

    def close(self):
        if getattr(self, "handle", None):
            _lib.bar_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class PeerRank:
    """One rank of separate processes without NCCL (bar_dist_create with nccl_id = NULL): the
    peer-memory async path only. ``allgather(obj) -> list`` exchanges small Python objects over
    any process group (tests: gloo); it carries the ghost lists and the CUDA IPC handles."""

    def __init__(self, A_rows, n_global, rows_per_block, device, rank, nranks, allgather, tuning=None):
        ranges = allgather((A_rows.row_lo, A_rows.row_hi))
        lo, hi = ghosts(A_rows)
        glists = allgather(np.concatenate([lo, hi]))
        rc, sc, si, gsrc = plan(rank, ranges, glists)
        self.handle = _create(n_global, A_rows, rows_per_block, device, nranks, rank, rc, sc, si, lo, hi, None)
        buf = ctypes.create_string_buffer(128)
        off = _i64()
        _check(_lib.bar_dist_p2p_handles(self.handle, buf, ctypes.byref(off)))
        allh = allgather((buf.raw, off.value))
        handles = ctypes.create_string_buffer(b"".join(h for h, _ in allh), 128 * nranks)
        offs = np.array([o for _, o in allh], dtype=np.int64)
        _check(_lib.bar_dist_enable_p2p(self.handle, _ptr(gsrc) if len(gsrc) else None, handles, _ptr(offs)))
        self.rank, self.nranks, self.n_local = rank, nranks, A_rows.row_hi - A_rows.row_lo
        if tuning:
            _check(_lib.bar_dist_set_tuning(self.handle, _tuning(tuning)))

    def solve(self, b, x0=None, x=None, k=5, max_global_iters=20000, tol=1e-10, mode="async", stream=None,
              raise_on_error=True):
        if x is None:
            import torch

            x = torch.empty_like(b) if hasattr(b, "data_ptr") else np.empty_like(b)
        info = SolveInfo()
        st = _lib.bar_dist_solve(self.handle, _ptr(b), _ptr(x0), _ptr(x), k, max_global_iters, tol, _mode(mode),
                                 _stream_handle(stream), ctypes.byref(info))
        if raise_on_error:
            _check(st)
        return x, _info(st, info)

    def close(self):
        if getattr(self, "handle", None):
            _lib.bar_dist_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class LoopbackGroup:
    """All ranks of a row partition in one process on one GPU (exchange = device copies)."""

    def __init__(self, blocks, n_global: int, rows_per_block: int, device: int = 0, tuning=None):
        P = len(blocks)
        ranges = [(A.row_lo, A.row_hi) for A in blocks]
        gh = [ghosts(A) for A in blocks]
        glists = [np.concatenate(g) for g in gh]
        self.handles = []
        for r, A in enumerate(blocks):
            rc, sc, si = make_plan(r, ranges, glists)
            self.handles.append(_create(n_global, A, rows_per_block, device, P, r, rc, sc, si, gh[r][0], gh[r][1],
                                        None))
        self._arr = (_vp * P)(*self.handles)
        _check(_lib.bar_dist_link_loopback(self._arr, P))
        self.ranges = ranges
        self.nranks = P
        self.ghost_cols = glists
        if tuning:
            for h in self.handles:
                _check(_lib.bar_dist_set_tuning(h, _tuning(tuning)))

    def enable_p2p(self):
        """Async mode pulls ghosts from the other ranks' live iterates (no exchange, no barrier)."""
        for r, h in enumerate(self.handles):
            src = ghost_sources(self.ranges, self.ghost_cols[r])
            _check(_lib.bar_dist_enable_p2p(h, _ptr(src) if len(src) else None, None, None))

    def solve(self, bs, x0s=None, xs=None, k=5, max_global_iters=20000, tol=1e-10, mode="async", stream=None,
              raise_on_error=True):
        P = self.nranks
        if xs is None:
            import torch

            xs = [torch.empty_like(b) for b in bs]
        arr = lambda vs: (_vp * P)(*[_ptr(v) for v in vs])  # noqa: E731
        info = SolveInfo()
        st = _lib.bar_dist_solve_loopback(self._arr, P, arr(bs), arr(x0s) if x0s is not None else None, arr(xs), k,
                                          max_global_iters, tol, _mode(mode), _stream_handle(stream),
                                          ctypes.byref(info))
        if raise_on_error:
            _check(st)
        return xs, _info(st, info)

    def close(self):
        for h in self.handles:
            _lib.bar_dist_destroy(h)
        self.handles = []

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


__all__ = ["ghosts", "localize", "partition", "plan", "make_plan", "ghost_sources", "nccl_unique_id", "DistMatrix",
           "PeerRank", "LoopbackGroup", "BarError"]

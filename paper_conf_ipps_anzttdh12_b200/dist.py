"""Multi-GPU row-partitioned solve: Python side of include/bar.h's ``bar_dist_*`` calls.

Marshalling and the process-group bookkeeping only (which rank owns which rows, who needs
whose rows); the exchange of x values, the sweeps and the residual run in libbar.so (NCCL
grouped send/recv + the block-sweep kernels). Paper: §3.4, SURVEY.md §8(e).

* ``ghosts``, ``localize`` — host planning through the C ABI (no GPU needed).
* ``make_plan`` — recv/send counts and send indices from every rank's ghost list.
* ``DistMatrix`` — one rank's share, created collectively over a torch.distributed group
  (NCCL transport; one process per GPU, launched with torchrun).
* ``LoopbackGroup`` — several ranks in one process on one GPU (device-to-device copies as the
  exchange): tests the partitioned path on a single B200.
"""
from __future__ import annotations

import ctypes

import numpy as np

from .bar import STATUS, BarError, SolveInfo, _check, _lib, _ptr, _stream_handle, MODES

_vp, _i64, _i32, _f64 = ctypes.c_void_p, ctypes.c_int64, ctypes.c_int32, ctypes.c_double
_lib.bar_dist_ghosts.restype = ctypes.c_int
_lib.bar_dist_ghosts.argtypes = [_i64, _i64, _i64, _vp, _vp, ctypes.POINTER(_i64), ctypes.POINTER(_i64), _vp]
_lib.bar_dist_localize.restype = ctypes.c_int
_lib.bar_dist_localize.argtypes = [_i64, _i64, _i64, _vp, _vp, _i64, _i64, _vp, _vp]
_lib.bar_nccl_unique_id.restype = ctypes.c_int
_lib.bar_nccl_unique_id.argtypes = [_vp]
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
_lib.bar_dist_destroy.restype = None
_lib.bar_dist_destroy.argtypes = [_vp]


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


def make_plan(rank: int, ranges, ghost_lists):
    """From every rank's (row range, sorted ghost list): this rank's recv_counts (per owner, in
    ghost order), send_counts and send_idx (owned local rows each peer needs, in its ghost order)."""
    P = len(ranges)
    starts = np.array([r[0] for r in ranges])
    ends = np.array([r[1] for r in ranges])

    def owner(cols):
        o = np.searchsorted(ends, cols, side="right")
        assert np.all((cols >= starts[o]) & (cols < ends[o]))
        return o

    mine = np.asarray(ghost_lists[rank], dtype=np.int64)
    recv_counts = np.bincount(owner(mine), minlength=P).astype(np.int64) if len(mine) else np.zeros(P, np.int64)
    send_counts = np.zeros(P, dtype=np.int64)
    send_idx = []
    b0, b1 = ranges[rank]
    for p in range(P):
        if p == rank:
            continue
        g = np.asarray(ghost_lists[p], dtype=np.int64)
        need = g[(g >= b0) & (g < b1)]
        send_counts[p] = len(need)
        send_idx.append((need - b0).astype(np.int32))
    send_idx = np.concatenate(send_idx) if send_idx else np.zeros(0, np.int32)
    return recv_counts, send_counts, np.ascontiguousarray(send_idx, dtype=np.int32)


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
    idbuf = None
    if nccl_id is not None:
        idbuf = ctypes.create_string_buffer(bytes(nccl_id), 128)
    _check(_lib.bar_dist_create(n_global, A_rows.row_lo, A_rows.row_hi, len(col_local), _ptr(rp), _ptr(col_local),
                                _ptr(val), len(lo), len(hi), nranks, rank, _ptr(recv_counts), _ptr(send_counts),
                                _ptr(send_idx), R, device, idbuf, ctypes.byref(h)))
    return h


def _info(st, info):
    d = info.as_dict()
    d["status"] = STATUS.get(st, st)
    return d


class DistMatrix:
    """This rank's share of a row-partitioned matrix (NCCL transport, one process per GPU)."""

    def __init__(self, A_rows, n_global: int, rows_per_block: int, device: int, group=None):
        import torch.distributed as dist

        P, r = dist.get_world_size(group), dist.get_rank(group)
        ranges = [None] * P
        dist.all_gather_object(ranges, (A_rows.row_lo, A_rows.row_hi), group=group)
        lo, hi = ghosts(A_rows)
        glists = [None] * P
        dist.all_gather_object(glists, np.concatenate([lo, hi]), group=group)
        recv_counts, send_counts, send_idx = make_plan(r, ranges, glists)
        nid = [None]
        if r == 0:
            buf = ctypes.create_string_buffer(128)
            _check(_lib.bar_nccl_unique_id(buf))
            nid[0] = buf.raw
        dist.broadcast_object_list(nid, src=0, group=group)
        self.handle = _create(n_global, A_rows, rows_per_block, device, P, r, recv_counts, send_counts, send_idx, lo,
                              hi, nid[0])
        self.rank, self.nranks, self.n_local = r, P, A_rows.row_hi - A_rows.row_lo
        self.row_lo, self.row_hi = A_rows.row_lo, A_rows.row_hi
        self.ranges, self.ghost_cols, self.group = ranges, np.concatenate([lo, hi]), group

    def enable_p2p(self):
        """Async over peer memory: exchange CUDA IPC handles of every rank's iterate and board."""
        import torch.distributed as dist

        buf = ctypes.create_string_buffer(128)
        off = _i64()
        _check(_lib.bar_dist_p2p_handles(self.handle, buf, ctypes.byref(off)))
        allh = [None] * self.nranks
        dist.all_gather_object(allh, (buf.raw, off.value), group=self.group)
        handles = ctypes.create_string_buffer(b"".join(h for h, _ in allh), 128 * self.nranks)
        offs = np.array([o for _, o in allh], dtype=np.int64)
        src = ghost_sources(self.ranges, self.ghost_cols)
        _check(_lib.bar_dist_enable_p2p(self.handle, _ptr(src), handles, _ptr(offs)))

    def solve(self, b, x0=None, x=None, k=5, max_global_iters=20000, tol=1e-10, mode="async", stream=None,
              raise_on_error=True):
        if x is None:
            import torch

            x = torch.empty_like(b) if hasattr(b, "data_ptr") else np.empty_like(b)
        info = SolveInfo()
        st = _lib.bar_dist_solve(self.handle, _ptr(b), _ptr(x0), _ptr(x), k, max_global_iters, tol,
                                 MODES[mode] if isinstance(mode, str) else mode, _stream_handle(stream),
                                 ctypes.byref(info))
        if raise_on_error:
            _check(st)
        return x, _info(st, info)

    def sweep(self, k=5, nsweeps=1, mode="async", stream=None):
        """Enqueue nsweeps local block-sweep launches (no exchange): kernel timing only."""
        _check(_lib.bar_dist_sweep(self.handle, k, nsweeps, MODES[mode] if isinstance(mode, str) else mode,
                                   _stream_handle(stream)))

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

    def __init__(self, blocks, n_global: int, rows_per_block: int, device: int = 0):
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

    def enable_p2p(self):
        """Async mode pulls ghosts from the other ranks' live iterates (no exchange, no barrier)."""
        for r, h in enumerate(self.handles):
            src = ghost_sources(self.ranges, self.ghost_cols[r])
            _check(_lib.bar_dist_enable_p2p(h, _ptr(src), None, None))

    def solve(self, bs, x0s=None, xs=None, k=5, max_global_iters=20000, tol=1e-10, mode="async", stream=None,
              raise_on_error=True):
        P = self.nranks
        if xs is None:
            import torch

            xs = [torch.empty_like(b) for b in bs]
        arr = lambda vs: (_vp * P)(*[_ptr(v) for v in vs])  # noqa: E731
        info = SolveInfo()
        st = _lib.bar_dist_solve_loopback(self._arr, P, arr(bs), arr(x0s) if x0s is not None else None, arr(xs), k,
                                          max_global_iters, tol, MODES[mode] if isinstance(mode, str) else mode,
                                          _stream_handle(stream), ctypes.byref(info))
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


__all__ = ["ghosts", "localize", "partition", "make_plan", "DistMatrix", "LoopbackGroup", "BarError"]

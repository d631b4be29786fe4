"""Multi-process (world size 2 and 3, gloo, CPU) tests of the multi-GPU host logic.

Each process owns a contiguous, subdomain-aligned row block. Through the C ABI's host-only
planning calls (bar_dist_ghosts / bar_dist_localize) and paper_conf_ipps_anzttdh12_b200.dist's
plan, the ranks exchange ghost lists and then the ghost VALUES over gloo (the NCCL exchange's
send/recv pattern), build the extended local vector [ghosts below | owned | ghosts above], and
run the ORACLE's sync-block / Jacobi step on the localized rows. The result must equal the
global one-process oracle step on those rows bit for bit: the local numbering is
order-preserving, so the per-row arithmetic is unchanged.
"""
import os
import socket
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, case, out_q):
    sys.path.insert(0, ROOT)
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    import torch
    import torch.distributed as dist

    import oracle as O
    import workloads as W
    from paper_conf_ipps_anzttdh12_b200 import dist as D

    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        kind, size, R, k = case
        gen = {"s7": W.stencil7_3d, "s9": W.stencil9_2d, "tref": W.trefethen}[kind]
        full = gen(size)
        n = full.n
        ranges = D.partition(n, R, world)
        b0, b1 = ranges[rank]
        A = gen(size, row_lo=b0, row_hi=b1)
        lo, hi = D.ghosts(A)
        # ghost lists: every rank's, through the process group
        glists = [None] * world
        dist.all_gather_object(glists, np.concatenate([lo, hi]))
        recv_counts, send_counts, send_idx = D.make_plan(rank, ranges, glists)
        # plan consistency: what p sends me is what I receive from p
        all_send = [None] * world
        dist.all_gather_object(all_send, send_counts.tolist())
        for p in range(world):
            assert all_send[p][rank] == recv_counts[p]
        col_local = D.localize(A, lo, hi)
        nglo = len(lo)
        # order preserved: each row's local columns ascend
        for i in range(b1 - b0):
            c = col_local[A.rowptr[i]:A.rowptr[i + 1]]
            assert np.all(np.diff(c) > 0)
        # the exchange: x_old is a seeded global vector; each rank only holds its own rows
        x_global = np.random.default_rng(3).uniform(-1, 1, n)
        b_global = np.ones(n)
        x_own = x_global[b0:b1].copy()
        send_buf = torch.from_numpy(x_own[send_idx].copy())
        off = np.concatenate([[0], np.cumsum(send_counts)])
        reqs, recv_bufs = [], {}
        for p in range(world):
            if p == rank:
                continue
            if send_counts[p]:
                reqs.append(dist.isend(send_buf[off[p]:off[p + 1]].contiguous(), dst=p))
            if recv_counts[p]:
                recv_bufs[p] = torch.empty(int(recv_counts[p]), dtype=torch.float64)
                reqs.append(dist.irecv(recv_bufs[p], src=p))
        for rq in reqs:
            rq.wait()
        ghosts_vals = np.concatenate([recv_bufs[p].numpy() for p in sorted(recv_bufs)]) if recv_bufs else np.zeros(0)
        x_ext = np.concatenate([ghosts_vals[:nglo], x_own, ghosts_vals[nglo:]])
        # the received values are the owners' values of my ghost columns
        assert np.array_equal(ghosts_vals, x_global[np.concatenate([lo, hi])])
        # oracle on the localized block: shift columns and rows by n_glo so indices are >= 0
        sub_global = []
        for TS in range(0, b1 - b0, R):
            TE = min(b1 - b0, TS + R)
            s, e = A.rowptr[TS], A.rowptr[TE]
            rows_loc = W.CSR(len(x_ext), A.rowptr[TS:TE + 1] - s, (col_local[s:e] + nglo).astype(np.int32),
                             A.val[s:e], nglo + TS, nglo + TE)
            if k == 0:
                y = O.jacobi_rows(rows_loc, b_global[b0 + TS:b0 + TE], x_ext)
            else:
                y = O.block_jacobi_subdomain(rows_loc, b_global[b0 + TS:b0 + TE], x_ext, k)
            sub_global.append(y)
        mine = np.concatenate(sub_global)
        if k == 0:
            ref = O.jacobi_step(full, b_global, x_global)[b0:b1]
        else:
            ref = O.block_jacobi_step(full, b_global, x_global, R, k)[b0:b1]
        out_q.put((rank, bool(np.array_equal(mine, ref)), float(np.abs(mine - ref).max())))
    except Exception as e:  # pragma: no cover
        out_q.put((rank, False, repr(e)))
    finally:
        dist.destroy_process_group()


CASES = [("s7", 10, 100, 5), ("s7", 9, 81, 0), ("s9", 30, 64, 3), ("tref", 1000, 128, 5)]


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("case", CASES)
def test_partitioned_step_bitwise(world, case):
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, ok, err in sorted(results):
        assert ok, (rank, err)


def test_partition_alignment():
    from paper_conf_ipps_anzttdh12_b200 import dist as D

    for n, R, P in [(1000, 100, 3), (134217728, 1024, 8), (2000, 128, 7), (10, 4, 4)]:
        rg = D.partition(n, R, P)
        assert rg[0][0] == 0 and rg[-1][1] == n
        for (a, b), (c, d) in zip(rg, rg[1:]):
            assert b == c and a % R == 0

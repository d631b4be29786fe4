"""The partitioned (multi-GPU) device path on ONE GPU: P loopback ranks in one process, the
exchange done by device-to-device copies (the NCCL path differs only in the transport call).

Sync-block and Jacobi iterates over P ranks must be bitwise identical to the one-GPU solve
(the order-preserving local numbering leaves every row's arithmetic unchanged), the stopping
iteration equal, and async must converge.
"""
import numpy as np
import pytest

import oracle as O
import workloads as W

pytestmark = pytest.mark.gpu


def _split(gen, args, n, R, P):
    from paper_conf_ipps_anzttdh12_b200 import dist as D

    return [gen(*args, row_lo=a, row_hi=b) for a, b in D.partition(n, R, P)]


def _single(bar, A, b, R, k, mode, iters, tol, x0, tuning=None):
    import torch

    M = bar.Matrix.from_csr(A, R, tuning=tuning)
    x = torch.empty(A.n, dtype=torch.float64, device="cuda")
    _, info = M.solve(torch.from_numpy(b).cuda(), torch.from_numpy(x0).cuda(), x, k=k, max_global_iters=iters,
                      tol=tol, mode=mode)
    M.close()
    return x.cpu().numpy(), info


def _loop(blocks, n, R, b, k, mode, iters, tol, x0, tuning=None):
    import torch

    from paper_conf_ipps_anzttdh12_b200 import dist as D

    G = D.LoopbackGroup(blocks, n, R, tuning=tuning)
    bs = [torch.from_numpy(b[a:c].copy()).cuda() for a, c in G.ranges]
    x0s = [torch.from_numpy(x0[a:c].copy()).cuda() for a, c in G.ranges]
    xs, info = G.solve(bs, x0s, None, k=k, max_global_iters=iters, tol=tol, mode=mode)
    G.close()
    return np.concatenate([x.cpu().numpy() for x in xs]), info


MATS = [("s7", W.stencil7_3d, (16,), 128), ("s9", W.stencil9_2d, (98,), 128), ("tref", W.trefethen, (2000,), 128),
        ("s7big", W.stencil7_3d, (64,), 1024)]


@pytest.mark.parametrize("name,gen,args,R", MATS)
@pytest.mark.parametrize("P", [1, 2, 3, 4])
@pytest.mark.parametrize("mode,k", [("sync-block", 5), ("jacobi", 1)])
def test_partitioned_iterates_bitwise(bar, name, gen, args, R, P, mode, k):
    A = gen(*args)
    n = A.n
    b = np.ones(n)
    x0 = np.random.default_rng(5).uniform(-1, 1, n)
    blocks = _split(gen, args, n, R, P)
    for m in (1, 4):
        xs, i1 = _single(bar, A, b, R, k, mode, m, 0.0, x0)
        xp, i2 = _loop(blocks, n, R, b, k, mode, m, 0.0, x0)
        assert np.array_equal(xs, xp), (m, np.abs(xs - xp).max())
        assert i2["iters"] == m
    # same stopping iteration at tol 1e-10; the returned iterate is the same bits
    xs, i1 = _single(bar, A, b, R, k, mode, 20000, 1e-10, np.zeros(n))
    xp, i2 = _loop(blocks, n, R, b, k, mode, 20000, 1e-10, np.zeros(n))
    assert i1["iters"] == i2["iters"] and i2["converged"]
    assert np.array_equal(xs, xp)
    assert abs(i1["rel_res"] - i2["rel_res"]) <= 1e-12 * i1["rel_res"]


@pytest.mark.parametrize("name,gen,args,R", MATS)
@pytest.mark.parametrize("P", [2, 4])
def test_partitioned_async_converges(bar, name, gen, args, R, P):
    A = gen(*args)
    n = A.n
    b = np.ones(n)
    blocks = _split(gen, args, n, R, P)
    x, info = _loop(blocks, n, R, b, 5, "async", 20000, 1e-10, np.zeros(n))
    assert info["converged"] and info["rel_res"] <= 1e-10
    assert O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)


@pytest.mark.parametrize("name,gen,args,R", MATS)
@pytest.mark.parametrize("P", [2, 4])
def test_partitioned_async_p2p(bar, name, gen, args, R, P):
    """Async over peer memory: ghosts pulled from the owners' live iterates, no halo exchange,
    no per-iteration collective; the result still meets the exact residual (by the oracle)."""
    import torch

    from paper_conf_ipps_anzttdh12_b200 import dist as D

    A = gen(*args)
    n = A.n
    b = np.ones(n)
    G = D.LoopbackGroup(_split(gen, args, n, R, P), n, R)
    G.enable_p2p()
    bs = [torch.from_numpy(b[a:c].copy()).cuda() for a, c in G.ranges]
    xs, info = G.solve(bs, None, None, k=5, mode="async")
    x = np.concatenate([v.cpu().numpy() for v in xs])
    G.close()
    assert info["converged"] and info["rel_res"] <= 1e-10
    assert O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)
    # no collective exchange inside the iteration: 3 launches per rank per global iteration
    # (pull, sweep, publish + estimate; 6 where the interior sweep overlaps the pull), plus the
    # confirming barriers / pull / residual
    assert info["iters"] > 0
    assert info["kernel_launches"] <= 6 * P * (info["iters"] + 12) + 16 * P, (info["kernel_launches"], info["iters"])


def test_plan_errors(bar):
    from paper_conf_ipps_anzttdh12_b200 import dist as D

    A = W.stencil7_3d(8)
    blk = W.stencil7_3d(8, row_lo=128, row_hi=256)
    lo, hi = D.ghosts(blk)
    z = np.zeros(2, dtype=np.int64)
    rc = np.array([len(lo), len(hi)], dtype=np.int64)
    idx = np.zeros(0, dtype=np.int32)
    with pytest.raises(D.BarError):  # row_begin = 128 is not a multiple of R = 96
        D._create(A.n, blk, 96, 0, 2, 1, rc[::-1].copy(), z, idx, lo, hi, None)
    with pytest.raises(D.BarError):  # a rank cannot receive from itself
        D._create(A.n, blk, 64, 0, 2, 1, np.array([0, len(lo) + len(hi)], dtype=np.int64), z, idx, lo, hi, None)


@pytest.mark.parametrize("P", [2, 3])
def test_partitioned_duo_coded(bar, P):
    """The two-blocks-per-SM kernel with coded columns on rank-local layouts (ghost columns below
    the owned block are negative local indices, the offsets d = col - row stay valid): sync-block
    and Jacobi bitwise the one-GPU iterates, async (chunked claims) converges."""
    tune = {"duo": 1}
    gen, args, R = W.stencil7_3d, (128,), 256  # two grid lines per subdomain: <= 4 local entries
    A = gen(*args)
    n = A.n
    b = np.ones(n)
    x0 = np.random.default_rng(7).uniform(-1, 1, n)
    blocks = _split(gen, args, n, R, P)
    for mode, k in (("sync-block", 5), ("jacobi", 1)):
        xs, _ = _single(bar, A, b, R, k, mode, 3, 0.0, x0, tuning=tune)
        xp, _ = _loop(blocks, n, R, b, k, mode, 3, 0.0, x0, tuning=tune)
        assert np.array_equal(xs, xp), mode
    x, info = _loop(blocks, n, R, b, 5, "async", 20000, 1e-10, np.zeros(n), tuning=tune)
    assert info["converged"] and O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)


@pytest.mark.parametrize("name,gen,args,R", MATS)
@pytest.mark.parametrize("P", [2, 3])
def test_halo_allgather_bitwise(bar, name, gen, args, R, P):
    """The ncclAllGather halo exchange (bar_tuning.halo = 1, SURVEY §8(e)'s primary design; here
    through the loopback transport's emulation of the gather): every rank's whole send buffer is
    gathered and each receiver copies its segments out, so sync-block and Jacobi iterates stay
    bitwise the one-GPU iterates, as with the grouped send/recv exchange."""
    tune = {"halo": "allgather"}
    A = gen(*args)
    n = A.n
    b = np.ones(n)
    x0 = np.random.default_rng(6).uniform(-1, 1, n)
    blocks = _split(gen, args, n, R, P)
    for mode, k in (("sync-block", 5), ("jacobi", 1)):
        xs, _ = _single(bar, A, b, R, k, mode, 3, 0.0, x0)
        xp, info = _loop(blocks, n, R, b, k, mode, 3, 0.0, x0, tuning=tune)
        assert np.array_equal(xs, xp), (mode, np.abs(xs - xp).max())
    x, info = _loop(blocks, n, R, b, 5, "async", 20000, 1e-10, np.zeros(n), tuning=tune)
    assert info["converged"] and O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)


# ------------------------------------------------------------------ bar_create_csr_dist over NCCL
@pytest.mark.parametrize("name,gen,args,R", MATS)
@pytest.mark.parametrize("halo", ["sendrecv", "allgather"])
def test_create_csr_dist_one_rank_nccl(bar, name, gen, args, R, halo):
    """§8(b)'s bar_create_csr_dist through the C ABI only (ctypes; no torch.distributed): a
    1-rank NCCL group (the box has one GPU). The library plans the share over NCCL (all-gathers
    of the row ranges, ghost counts, devices and ghost lists; a min all-reduce of the peer-access
    flags; an all-gather of the IPC handles), and the solve runs the collective path
    (ncclGroupStart/End of the halo exchange or an in-place ncclAllGather, an ncclAllGather of the
    residual partials per iteration): sync-block and Jacobi iterates and iteration counts are
    bitwise those of bar_solve; async runs the peer-memory path (board barriers with itself)."""
    import ctypes

    import torch

    from paper_conf_ipps_anzttdh12_b200 import dist as D

    A = gen(*args)
    n = A.n
    b = np.ones(n)
    x0 = np.random.default_rng(8).uniform(-1, 1, n)
    nid = ctypes.create_string_buffer(128)
    assert bar._lib.bar_nccl_unique_id(nid) == 0, bar.bar_last_error()
    h = ctypes.c_void_p()
    rp, col, val = (np.ascontiguousarray(a) for a in (A.rowptr, A.col, A.val))
    st = bar._lib.bar_create_csr_dist(n, 0, n, A.nnz, rp.ctypes.data, col.ctypes.data, val.ctypes.data, R, 0, nid, 0,
                                      1, ctypes.byref(h))
    assert st == 0, bar.bar_last_error()
    bar.bar_set_tuning(h, {"halo": halo})
    bd, x0d = torch.from_numpy(b).cuda(), torch.from_numpy(x0).cuda()
    for mode, k in (("sync-block", 5), ("jacobi", 1)):
        for m, tol in ((3, 0.0), (20000, 1e-10)):
            xs, i1 = _single(bar, A, b, R, k, mode, m, tol, x0)
            xd = torch.empty_like(bd)
            _, i2 = bar.bar_solve(h, bd, x0d, xd, k, m, tol, mode)
            assert np.array_equal(xs, xd.cpu().numpy()), (mode, m)
            assert i1["iters"] == i2.iters
    xd = torch.empty_like(bd)
    _, info = bar.bar_solve(h, bd, None, xd, 5, 20000, 1e-10, "async")
    assert info.converged and O.rel_res(A, b, xd.cpu().numpy()) <= 1e-10 * (1 + 1e-6)
    r, bn = bar.bar_residual(h, bd, xd)
    ref = O.rel_res(A, b, xd.cpu().numpy())  # b - A x cancels near convergence: DESIGN.md R16
    assert abs(r / bn - ref) <= 1e-6 * ref + 1e-15, (r / bn, ref)
    # bar_sweep on the share: local launches (one rank: the whole matrix), oracle's iterates
    xd = x0d.clone()
    bar.bar_sweep(h, bd, xd, 5, 2, "sync-block")
    torch.cuda.synchronize()
    ref = O.block_jacobi_step(A, b, O.block_jacobi_step(A, b, x0, R, 5), R, 5)
    assert np.abs(xd.cpu().numpy() - ref).max() <= 1e-12 * np.abs(ref).max()
    bar.bar_destroy(h)
    # the Python wrapper (marshalling only) over the same call
    M = D.DistMatrix(A, n, R, 0, D.nccl_unique_id(), 0, 1)
    xm, info = M.solve(bd, None, None, k=5, mode="sync-block")
    xs, i1 = _single(bar, A, b, R, 5, "sync-block", 20000, 1e-10, np.zeros(n))
    assert np.array_equal(xs, xm.cpu().numpy()) and info["iters"] == i1["iters"]
    M.close()


def test_create_csr_dist_errors(bar):
    import ctypes

    from paper_conf_ipps_anzttdh12_b200 import dist as D  # noqa: F401  (sets the argtypes)

    A = W.stencil7_3d(8)
    rp, col, val = (np.ascontiguousarray(a) for a in (A.rowptr, A.col, A.val))
    nid = ctypes.create_string_buffer(128)
    assert bar._lib.bar_nccl_unique_id(nid) == 0
    h = ctypes.c_void_p()
    # no NCCL id
    assert bar._lib.bar_create_csr_dist(A.n, 0, A.n, A.nnz, rp.ctypes.data, col.ctypes.data, val.ctypes.data, 64, 0,
                                        None, 0, 1, ctypes.byref(h)) == 1
    # row_begin not a multiple of R
    blk = W.stencil7_3d(8, row_lo=100, row_hi=200)
    brp, bcol, bval = (np.ascontiguousarray(a) for a in (blk.rowptr, blk.col, blk.val))
    assert bar._lib.bar_create_csr_dist(A.n, 100, 200, blk.nnz, brp.ctypes.data, bcol.ctypes.data, bval.ctypes.data,
                                        64, 0, nid, 0, 2, ctypes.byref(h)) == 1
    # a column outside [0, n_global)
    bad = col.copy()
    bad[5] = A.n + 3
    assert bar._lib.bar_create_csr_dist(A.n, 0, A.n, A.nnz, rp.ctypes.data, bad.ctypes.data, val.ctypes.data, 64, 0,
                                        nid, 0, 1, ctypes.byref(h)) == 2


# ------------------------------------------------------------------ separate processes, peer memory
def _peer_worker(rank, world, store, case, q):
    import os
    import sys

    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import numpy as np
    import torch
    import torch.distributed as dist

    import workloads as W
    from paper_conf_ipps_anzttdh12_b200 import dist as D

    torch.cuda.set_device(0)
    # a file store (no TCP port to race for); gloo only carries the ghost lists and IPC handles
    dist.init_process_group("gloo", init_method=f"file://{store}", rank=rank, world_size=world)
    try:
        kind, size, R, k = case
        gen = {"s7": W.stencil7_3d, "s9": W.stencil9_2d, "tref": W.trefethen}[kind]
        n = gen(size).n
        a, c = D.partition(n, R, world)[rank]
        A = gen(size, row_lo=a, row_hi=c)

        def allgather(o):
            out = [None] * world
            dist.all_gather_object(out, o)
            return out

        Pr = D.PeerRank(A, n, R, 0, rank, world, allgather)
        b = torch.ones(c - a, dtype=torch.float64, device="cuda")
        outs = []
        for _ in range(2):  # twice: epochs and stop tags carry over between solves
            x, info = Pr.solve(b, None, None, k=k, tol=1e-10, mode="async")
            outs.append((x.cpu().numpy(), info))
        Pr.close()
        q.put((rank, outs))
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("case", [("s7", 24, 128, 5), ("tref", 2000, 128, 5), ("s9", 98, 128, 2)])
@pytest.mark.parametrize("world", [2, 3])
def test_peer_processes_one_gpu(bar, case, world):
    """The peer-memory async mode with SEPARATE PROCESSES sharing the one GPU: real CUDA IPC
    mappings of every rank's iterate and board (handles exchanged over gloo), ghost pulls with
    relaxed system-scope loads, stop requests through the boards, and the confirming residual
    behind two board barriers — no NCCL, no collective while iterating. Every rank returns
    converged with the same exact residual; the assembled x meets it by the oracle."""
    import multiprocessing as mp
    import tempfile

    import workloads as W

    store = tempfile.mktemp(prefix="bar_peer_store_")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_peer_worker, args=(r, world, store, case, q), daemon=True) for r in range(world)]
    for p in ps:
        p.start()
    try:
        res = dict(q.get(timeout=240) for _ in ps)
    finally:
        for p in ps:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    for r in range(world):
        assert not isinstance(res[r], str), res[r]
    kind, size, R, k = case
    gen = {"s7": W.stencil7_3d, "s9": W.stencil9_2d, "tref": W.trefethen}[kind]
    A = gen(size)
    b = np.ones(A.n)
    for s_ in range(2):
        infos = [res[r][s_][1] for r in range(world)]
        x = np.concatenate([res[r][s_][0] for r in range(world)])
        for i in infos:
            assert i["converged"] and i["rel_res"] <= 1e-10, i
        assert len({i["rel_res"] for i in infos}) == 1  # the same bits on every rank
        assert len({i["iters"] for i in infos}) == 1  # min over ranks, agreed through the boards
        assert O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)


@pytest.mark.parametrize("name,gen,args,R", [("s7big", W.stencil7_3d, (64,), 1024), ("s7", W.stencil7_3d, (16,), 128),
                                             ("s9", W.stencil9_2d, (200,), 512)])
@pytest.mark.parametrize("P", [2, 3])
@pytest.mark.parametrize("mode,k", [("sync-block", 5), ("jacobi", 1), ("async", 5)])
def test_interior_boundary_overlap(bar, name, gen, args, R, P, mode, k):
    """SURVEY §8(e)'s overlap on the collective path: each rank sweeps its interior subdomains
    (no ghost column) on a second stream while the halo exchange runs, then its boundary
    subdomains. Sync-block and Jacobi iterates are bitwise those without the overlap (and of
    the one-GPU solve); async converges; the overlapped path really ran (more launches: three
    sweep launches and a partial-sum kernel per rank and iteration)."""
    A = gen(*args)
    n = A.n
    b = np.ones(n)
    x0 = np.random.default_rng(19).uniform(-1, 1, n)
    blocks = _split(gen, args, n, R, P)
    if mode == "async":
        x, i_on = _loop(blocks, n, R, b, k, mode, 20000, 1e-10, np.zeros(n))
        assert i_on["converged"] and O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)
        return
    xs, _ = _single(bar, A, b, R, k, mode, 4, 0.0, x0)
    x_on, i_on = _loop(blocks, n, R, b, k, mode, 4, 0.0, x0)
    x_off, i_off = _loop(blocks, n, R, b, k, mode, 4, 0.0, x0, tuning={"overlap": -1})
    assert np.array_equal(x_on, x_off) and np.array_equal(x_on, xs)
    if mode == "sync-block":  # Jacobi at R = 128 runs a kernel without subdomain ranges: no overlap
        assert i_on["kernel_launches"] > i_off["kernel_launches"], (i_on, i_off)
    _, c_on = _loop(blocks, n, R, b, k, mode, 20000, 1e-10, np.zeros(n))
    _, c_off = _loop(blocks, n, R, b, k, mode, 20000, 1e-10, np.zeros(n), tuning={"overlap": -1})
    assert c_on["iters"] == c_off["iters"] and c_on["converged"]


def _absent_worker(rank, world, store, q):
    import os
    import sys
    import time

    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch
    import torch.distributed as dist

    import workloads as W
    from paper_conf_ipps_anzttdh12_b200 import dist as D

    torch.cuda.set_device(0)
    dist.init_process_group("gloo", init_method=f"file://{store}", rank=rank, world_size=world)
    try:
        n = W.stencil7_3d(16).n
        a, c = D.partition(n, 128, world)[rank]
        A = W.stencil7_3d(16, row_lo=a, row_hi=c)

        def allgather(o):
            out = [None] * world
            dist.all_gather_object(out, o)
            return out

        Pr = D.PeerRank(A, n, 128, 0, rank, world, allgather)
        if rank == 0:
            t0 = time.time()
            b = torch.ones(c - a, dtype=torch.float64, device="cuda")
            _, info = Pr.solve(b, mode="async", raise_on_error=False)
            q.put((rank, info["status"], time.time() - t0))
            dist.barrier()
        else:  # rank 1 never joins the solve; it keeps its memory mapped until rank 0 is done
            q.put((rank, "absent", 0.0))
            dist.barrier()
        Pr.close()
    except Exception as e:  # pragma: no cover
        q.put((rank, repr(e), 0.0))
    finally:
        dist.destroy_process_group()


def test_peer_timeout_when_a_rank_is_absent(bar):
    """A rank that never joins a peer-memory solve makes the others fail with BAR_ERR_NCCL after the
    board barrier's 20 s timeout — no hang, no device fault (the GPU stays usable)."""
    import multiprocessing as mp
    import tempfile

    store = tempfile.mktemp(prefix="bar_absent_store_")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_absent_worker, args=(r, 2, store, q), daemon=True) for r in range(2)]
    for p in ps:
        p.start()
    try:
        res = {r: (st, dt) for r, st, dt in (q.get(timeout=120) for _ in ps)}
    finally:
        for p in ps:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    assert res[1][0] == "absent"
    assert res[0][0] == "BAR_ERR_NCCL", res
    assert 15 < res[0][1] < 60, res


@pytest.mark.parametrize("P", [2, 3])
def test_peer_memory_overlap(bar, P):
    """Async over peer memory with the interior subdomains swept on a second stream while the
    ghosts are pulled (then the boundary ones): converges to the exact residual like the serial
    pull-then-sweep order, and the overlapped order really ran (more launches per iteration)."""
    import torch

    from paper_conf_ipps_anzttdh12_b200 import dist as D

    gen, args, R = W.stencil7_3d, (64,), 1024
    A = gen(*args)
    n = A.n
    b = np.ones(n)
    out = {}
    for ov in (0, -1):
        G = D.LoopbackGroup(_split(gen, args, n, R, P), n, R, tuning={"overlap": ov})
        G.enable_p2p()
        bs = [torch.from_numpy(b[a:c].copy()).cuda() for a, c in G.ranges]
        xs, info = G.solve(bs, None, None, k=5, mode="async")
        x = np.concatenate([v.cpu().numpy() for v in xs])
        G.close()
        assert info["converged"] and O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6), (ov, info)
        out[ov] = info
    per_it = {ov: out[ov]["kernel_launches"] / max(1, out[ov]["cta_iters_max"]) for ov in out}
    assert per_it[0] > per_it[-1], out

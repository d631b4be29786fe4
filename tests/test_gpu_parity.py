"""GPU parity: the CUDA path (through libbar.so's C ABI) against the CPU oracle.

Tolerances: sync-block and Jacobi iterates must match the oracle to
||x_gpu - x_oracle||_inf <= 1e-12 * ||x_oracle||_inf at every checked iterate (north star);
exact (dyadic) cases bitwise; iteration counts equal. Async is nondeterministic (eq. 3,
P:93-99) and is validated by outcome: exact rel_res <= tol, solution within 1e-8 relative of
the direct solve, iteration count reported next to the oracle's.
"""
import numpy as np
import pytest

import oracle as O
import workloads as W

pytestmark = pytest.mark.gpu

TOL_ITERATE = 1e-12


def _dev(a):
    import torch

    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _solve(bar, A, b, R, k, mode, max_iters, tol, x0=None, tuning=None):
    import torch

    M = bar.Matrix.from_csr(A, rows_per_block=R, tuning=tuning)
    bd = _dev(b)
    x0d = None if x0 is None else _dev(x0)
    x = torch.empty_like(bd)
    x, info = M.solve(bd, x0d, x, k=k, max_global_iters=max_iters, tol=tol, mode=mode)
    torch.cuda.synchronize()
    M.close()
    return x.cpu().numpy(), info


def _close(x, ref, tol=TOL_ITERATE):
    err = np.abs(x - ref).max()
    scale = np.abs(ref).max()
    assert err <= tol * scale, (err, scale, err / scale)


MATS = {
    "tref2000": lambda: W.trefethen(2000),
    "fv1": lambda: W.stencil9_2d(98),
    "s7_m12": lambda: W.stencil7_3d(12),
    "rand": lambda: W.random_dd(3001, 7, seed=11, symmetric_pattern=True),
}


# ------------------------------------------------------------------ boundary errors
def test_create_errors(bar):
    A = W.trefethen(64)
    rp, c, v = A.rowptr.copy(), A.col.copy(), A.val.copy()

    def st(rp, c, v, R=16, n=64):
        with pytest.raises(bar.BarError) as e:
            bar.bar_create_csr(n, int(rp[-1]), rp, c, v, R)
        return e.value.name

    bad = rp.copy(); bad[0] = 1
    assert st(bad, c, v) == "BAR_ERR_BAD_CSR"
    bad = c.copy(); bad[5] = 64
    assert st(rp, bad, v) == "BAR_ERR_BAD_CSR"
    bad = c.copy(); bad[[3, 4]] = bad[[4, 3]]
    assert st(rp, bad, v) == "BAR_ERR_BAD_CSR"
    dv = v.copy(); dv[rp[0] + np.searchsorted(c[rp[0]:rp[1]], 0)] = 0.0
    assert st(rp, c, dv) == "BAR_ERR_ZERO_DIAG"
    nv = v.copy(); nv[7] = np.nan
    assert st(rp, c, nv) == "BAR_ERR_NONFINITE"
    assert st(rp, c, v, R=0) == "BAR_ERR_INVALID_ARG"
    assert st(rp, c, v, R=bar.MAX_ROWS_PER_BLOCK + 1) == "BAR_ERR_INVALID_ARG"
    # missing diagonal in row 0
    D = A.to_dense(); D[0, 0] = 0
    nz = [np.nonzero(D[i])[0] for i in range(64)]
    rp2 = np.concatenate([[0], np.cumsum([len(z) for z in nz])]).astype(np.int32)
    c2 = np.concatenate(nz).astype(np.int32)
    v2 = np.concatenate([D[i, z] for i, z in enumerate(nz)])
    assert st(rp2, c2, v2) == "BAR_ERR_BAD_CSR"


def test_solve_arg_errors(bar):
    import torch

    A = W.trefethen(100)
    M = bar.Matrix.from_csr(A, 32)
    b = torch.ones(100, dtype=torch.float64, device="cuda")
    for kw in ({"k": 0, "mode": "async"}, {"tol": -1.0}, {"tol": float("nan")}, {"max_global_iters": -1}):
        args = dict(k=5, max_global_iters=10, tol=1e-10, mode="sync-block")
        args.update(kw)
        with pytest.raises(bar.BarError) as e:
            M.solve(b, **args)
        assert e.value.name == "BAR_ERR_INVALID_ARG"
    bn = b.clone(); bn[3] = float("inf")
    for mode in ("async", "sync-block", "jacobi"):
        with pytest.raises(bar.BarError) as e:
            M.solve(bn, mode=mode)
        assert e.value.name == "BAR_ERR_NONFINITE"


# ------------------------------------------------------------------ residual
@pytest.mark.parametrize("name", list(MATS))
@pytest.mark.parametrize("R", [1, 37, 128, 1000])
def test_residual_parity(bar, name, R):
    A = MATS[name]()
    rng = np.random.default_rng(R)
    x = rng.standard_normal(A.n)
    b = rng.standard_normal(A.n)
    M = bar.Matrix.from_csr(A, R)
    r, bn = M.residual(_dev(b), _dev(x))
    ref = O.residual_norm(A, b, x)
    assert abs(r - ref) <= 1e-13 * ref
    assert abs(bn - O.norm2(b)) <= 1e-14 * bn
    # host pointers (end-to-end path) give the same bits
    r2, bn2 = M.residual(b, x)
    assert r2 == r and bn2 == bn


# ------------------------------------------------------------------ iterate-by-iterate
@pytest.mark.parametrize("name", list(MATS))
@pytest.mark.parametrize("mode,k,R", [("jacobi", 1, 128), ("sync-block", 1, 128), ("sync-block", 2, 100),
                                      ("sync-block", 5, 128), ("sync-block", 5, 448), ("sync-block", 9, 1024),
                                      ("sync-block", 3, 1), ("sync-block", 5, 8192), ("sync-block", 4, 4000),
                                      ("sync-block", 5, 99), ("sync-block", 2, 256), ("sync-block", 5, 512)])
def test_iterates_match_oracle(bar, name, mode, k, R):
    A = MATS[name]()
    b = np.ones(A.n)
    x0 = np.random.default_rng(1).uniform(-1, 1, A.n)
    checks = [1, 2, 3, 7, 15]
    ref = x0.copy()
    refs = {}
    for m in range(1, max(checks) + 1):
        ref = O.jacobi_step(A, b, ref) if mode == "jacobi" else O.block_jacobi_step(A, b, ref, R, k)
        refs[m] = ref
    for m in checks:
        x, info = _solve(bar, A, b, R, k, mode, m, 0.0, x0)
        assert info["iters"] == m and info["converged"] == 0
        _close(x, refs[m])
        assert abs(info["rel_res"] - O.rel_res(A, b, refs[m])) <= 1e-9 * info["rel_res"] + 1e-15


@pytest.mark.parametrize("name,mode,k,R", [("tref2000", "jacobi", 1, 128), ("tref2000", "sync-block", 5, 128),
                                           ("tref2000", "sync-block", 9, 128), ("fv1", "sync-block", 5, 128),
                                           ("fv1", "sync-block", 5, 448), ("fv1", "jacobi", 1, 448),
                                           ("s7_m12", "sync-block", 2, 288), ("rand", "sync-block", 5, 256)])
def test_iteration_count_and_solution(bar, name, mode, k, R):
    """Same stopping iteration as the oracle (O5), same returned iterate to 1e-12."""
    A = MATS[name]()
    b = np.ones(A.n)
    meth = O.JACOBI if mode == "jacobi" else O.BLOCK_JACOBI
    r = O.solve(A, b, method=meth, R=R, k=k, tol=1e-10)
    x, info = _solve(bar, A, b, R, k, mode, 20000, 1e-10)
    assert info["converged"] == 1 and info["iters"] == r.iters
    assert info["rel_res"] <= 1e-10
    _close(x, r.x)


@pytest.mark.parametrize("mode,k,R", [("jacobi", 1, 448), ("sync-block", 5, 128)])
def test_few_launches_queued_past_the_stop(bar, mode, k, R):
    """The per-launch solve loop sizes its last chunk from the observed residual rate
    (ChunkSizer, csrc/bar_internal.cuh): on fv1 (Jacobi 146, sync-block-(5) 92 iterations) doubling
    chunks 8, 16, 32, 64, 128 would queue 248 / 120 sweeps; the sized chunk stays within a few
    launches of iters + 1 (the stop is detected in the sweep after x^(iters)). Same iterate and
    count as the oracle either way."""
    A = MATS["fv1"]()
    b = np.ones(A.n)
    meth = O.JACOBI if mode == "jacobi" else O.BLOCK_JACOBI
    r = O.solve(A, b, method=meth, R=R, k=k, tol=1e-10)
    x, info = _solve(bar, A, b, R, k, mode, 20000, 1e-10)
    assert info["converged"] == 1 and info["iters"] == r.iters
    _close(x, r.x)
    assert info["kernel_launches"] <= r.iters + 1 + 12, (info["kernel_launches"], r.iters)


def test_dyadic_bitwise(bar):
    """Exact dyadic iterates: GPU == oracle bit for bit, any order/FMA."""
    A = W.dyadic_stencil9_2d(40, p=4)
    b = (np.arange(A.n) % 5 - 2).astype(float)
    # exact while the total number of sweeps m*k stays <= ~50/p = 12 (denominators 2^(4 m k))
    for mode, k, R, ms in [("jacobi", 1, 64, (1, 5, 12)), ("sync-block", 3, 64, (1, 2, 4)),
                           ("sync-block", 2, 100, (1, 3, 6))]:
        for m in ms:
            x, _ = _solve(bar, A, b, R, k, mode, m, 0.0)
            ref = np.zeros(A.n)
            for _ in range(m):
                ref = O.jacobi_step(A, b, ref) if mode == "jacobi" else O.block_jacobi_step(A, b, ref, R, k)
            assert np.array_equal(x, ref)


def test_sync_modes_bitwise_reproducible(bar):
    A = W.trefethen(20000)
    b = np.ones(A.n)
    for mode in ("sync-block", "jacobi"):
        x1, i1 = _solve(bar, A, b, 128, 5, mode, 20000, 1e-10)
        x2, i2 = _solve(bar, A, b, 128, 5, mode, 20000, 1e-10)
        assert np.array_equal(x1, x2) and i1["iters"] == i2["iters"] and i1["rel_res"] == i2["rel_res"]


def test_host_pointers_end_to_end(bar):
    """The end-to-end path (host b/x0/x, copies inside the call) gives the device path's bits."""
    import torch

    A = W.stencil9_2d(98)
    M = bar.Matrix.from_csr(A, 448)
    b = np.ones(A.n)
    xh = np.empty(A.n)
    _, ih = M.solve(b, None, xh, k=5, mode="sync-block")
    xd, idd = M.solve(_dev(b), None, None, k=5, mode="sync-block")
    torch.cuda.synchronize()
    assert np.array_equal(xh, xd.cpu().numpy()) and ih["iters"] == idd["iters"]
    # x may alias x0
    x = _dev(np.zeros(A.n))
    M.solve(_dev(b), x, x, k=5, mode="sync-block")
    assert np.array_equal(x.cpu().numpy(), xh)


# ------------------------------------------------------------------ special cases
def test_b_zero_and_converged_start(bar):
    A = W.trefethen(500)
    x, info = _solve(bar, A, np.zeros(500), 128, 5, "async", 100, 1e-10, x0=np.ones(500))
    assert info["iters"] == 0 and info["converged"] and np.all(x == 0)
    xs = np.linalg.solve(A.to_dense(), np.ones(500))
    for mode in ("async", "sync-block", "jacobi"):
        x, info = _solve(bar, A, np.ones(500), 128, 5, mode, 100, 1e-10, x0=xs)
        assert info["iters"] == 0 and info["converged"] and np.array_equal(x, xs)


def test_zero_start_shortcut(bar):
    """x0 = NULL (zero start): the exact residual of x^(0) is ||b|| / ||b|| = 1 without an SpMV
    (b = 0: x = 0 returned at once); the solve is the same as with an explicit zero x0."""
    A = W.trefethen(500)
    x, info = _solve(bar, A, np.zeros(500), 128, 5, "async", 100, 1e-10)
    assert info["iters"] == 0 and info["converged"] and np.all(x == 0)
    x1, i1 = _solve(bar, A, np.ones(500), 128, 5, "async", 0, 1e-10)
    assert i1["iters"] == 0 and not i1["converged"] and i1["rel_res"] == 1.0 and np.all(x1 == 0)
    x2, i2 = _solve(bar, A, np.ones(500), 128, 5, "async", 20000, 1e-10)
    assert i2["converged"] and O.rel_res(A, np.ones(500), x2) <= 1e-10 * (1 + 1e-6)


@pytest.mark.parametrize("mode", ["async", "sync-block", "jacobi"])
def test_fixed_point_invariant(bar, mode):
    """Starting at x* with tol = 0, every mode (async included) stays at x* (P7)."""
    A = W.trefethen(2000)
    b = np.ones(A.n)
    xs = np.linalg.solve(A.to_dense(), b)
    x, info = _solve(bar, A, b, 128, 5, mode, 12, 0.0, x0=xs)
    assert info["iters"] == 12
    assert np.abs(x - xs).max() <= 1e-14 * np.abs(xs).max() * 10


@pytest.mark.parametrize("mode", ["sync-block", "jacobi"])
def test_divergence(bar, mode):
    """rho(B) = 1.8 > 1 (P:697 analogue, SPD): the synchronous iterations diverge -> BAR_ERR_DIVERGED."""
    Ad = np.full((3, 3), 0.9) + 0.1 * np.eye(3)
    A = W.CSR(3, np.array([0, 3, 6, 9], dtype=np.int32), np.tile(np.arange(3, dtype=np.int32), 3), Ad.ravel())
    M = bar.Matrix.from_csr(A, 1)
    b = _dev(np.ones(3))
    _, info = M.solve(b, k=1, mode=mode, raise_on_error=False)
    assert info["status"] == "BAR_ERR_DIVERGED"


def test_divergence_async(bar):
    """Async with rho(|B|) >= 1 (Chazan-Miranker): only SOME update orders must diverge —
    the SPD 3x3 case above converges under Gauss-Seidel-like orders, so which one a schedule
    produces is not fixed. A = [[1, 2], [2, 1]] diverges under EVERY order: each update sets
    e_i = -2 e_j, doubling the error, so async-(k) must return BAR_ERR_DIVERGED."""
    A = W.CSR(2, np.array([0, 2, 4], dtype=np.int32), np.array([0, 1, 0, 1], dtype=np.int32),
              np.array([1.0, 2.0, 2.0, 1.0]))
    for R in (1, 2):
        M = bar.Matrix.from_csr(A, R)
        _, info = M.solve(_dev(np.ones(2)), k=1, mode="async", raise_on_error=False)
        assert info["status"] == "BAR_ERR_DIVERGED", (R, info)


# ------------------------------------------------------------------ async outcome
@pytest.mark.parametrize("name,k,R,envelope", [("tref2000", 5, 128, (15, 35)), ("tref2000", 1, 128, (60, 160)),
                                               ("fv1", 5, 128, (40, 110)), ("fv1", 2, 448, (30, 120)),
                                               ("rand", 5, 256, (2, 200)), ("s7_m12", 9, 288, (2, 200))])
def test_async_outcome(bar, name, k, R, envelope):
    """async-(k): exact rel_res <= 1e-10, x within 1e-8 (relative) of the direct solve,
    iteration count inside the envelope around the oracle's sync-block count (P5, Table 3)."""
    A = MATS[name]()
    b = np.ones(A.n)
    xs = np.linalg.solve(A.to_dense(), b)
    x, info = _solve(bar, A, b, R, k, "async", 20000, 1e-10)
    assert info["converged"] == 1 and info["rel_res"] <= 1e-10
    assert O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)
    assert np.abs(x - xs).max() <= 1e-8 * np.abs(xs).max()
    assert envelope[0] <= info["iters"] <= envelope[1], info["iters"]


def test_async_c3_against_cg(bar):
    """C3 (Trefethen_20000) with b = 1 at the bench configuration (async-(5), R = 128, tol 1e-10)
    against a host CG solve to 1e-15 (Jacobi-preconditioned, scipy): ||x - x*||_inf <= 1e-8
    ||x*||_inf (P6; cond_2 ~ 1.5e4 here, so the residual alone would not imply it)."""
    import scipy.sparse.linalg as spla

    A = W.trefethen(20000)
    b = np.ones(A.n)
    S = A.to_scipy()
    dinv = 1.0 / S.diagonal()
    Mp = spla.LinearOperator(S.shape, matvec=lambda v: dinv * v)
    xs, rc = spla.cg(S, b, rtol=1e-15, atol=0.0, maxiter=5000, M=Mp)
    assert rc == 0 and np.linalg.norm(b - S @ xs) <= 1e-13 * np.linalg.norm(b)
    x, info = _solve(bar, A, b, 128, 5, "async", 20000, 1e-10)
    assert info["converged"] and O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)
    assert np.abs(x - xs).max() <= 1e-8 * np.abs(xs).max()
    assert 15 <= info["iters"] <= 35, info["iters"]  # the oracle's sync-block-(5): 26 (P12)


@pytest.mark.parametrize("name,R", [("tref2000", 128), ("fv1", 448), ("s7_m12", 288), ("rand", 1024)])
@pytest.mark.parametrize("mode,k", [("sync-block", 5), ("jacobi", 1), ("sync-block", 2)])
def test_bar_sweep_matches_oracle(bar, name, R, mode, k):
    """bar_sweep (no convergence control; the per-launch timing entry point of bench.py and N4)
    leaves exactly nsweeps oracle steps in x, for odd and even nsweeps (the sync modes ping-pong
    between x and the library buffer)."""
    import torch

    A = MATS[name]()
    b = np.ones(A.n)
    x0 = np.random.default_rng(17).uniform(-1, 1, A.n)
    M = bar.Matrix.from_csr(A, R)
    bd = _dev(b)
    for nsw in (1, 2, 5):
        xd = _dev(x0)
        M.sweep(bd, xd, k=k, nsweeps=nsw, mode=mode)
        torch.cuda.synchronize()
        ref = x0
        for _ in range(nsw):
            ref = O.jacobi_step(A, b, ref) if mode == "jacobi" else O.block_jacobi_step(A, b, ref, R, k)
        _close(xd.cpu().numpy(), ref)
    M.close()


@pytest.mark.parametrize("name,R,single", [("tref2000", 128, 1), ("tref2000", 128, -1), ("fv1", 448, -1),
                                            ("s7_m12", 288, -1)])
def test_bar_sweep_async_does_the_work(bar, name, R, single):
    """bar_sweep in async mode runs nsweeps global iterations: after N sweeps from x0 = 0 the
    exact residual is within a factor 30 of what N oracle sync-block-(5) iterations leave (the
    async order is at least as fast as sync-block's, P5/R15), and it keeps shrinking with N —
    a sweep that did less work would show up here (and would inflate the bench's per-launch
    timing)."""
    import torch

    A = MATS[name]()
    b = np.ones(A.n)
    M = bar.Matrix.from_csr(A, R, tuning={"single_launch": single})
    bd = _dev(b)
    prev = None
    for nsw in (4, 12):
        xd = torch.zeros(A.n, dtype=torch.float64, device="cuda")
        M.sweep(bd, xd, k=5, nsweeps=nsw, mode="async")
        torch.cuda.synchronize()
        rr = O.rel_res(A, b, xd.cpu().numpy())
        ref = O.solve(A, b, method=O.BLOCK_JACOBI, R=R, k=5, tol=0.0, max_iters=nsw).rel_res
        assert rr <= 30 * ref, (nsw, rr, ref)
        if prev is not None:  # 8 more global iterations (each contracts by well under 0.75 here)
            assert rr < 0.1 * prev, (rr, prev)
        prev = rr
    M.close()


def test_siam_constant_async(bar, golden):
    """Trefethen_20000, b = e_1: x_1 = (A^-1)_11 = 0.7250783462684011674...."""
    ref = float(golden("siam_trefethen20000_a11.txt")[0][0])
    A = W.trefethen(20000)
    b = np.zeros(A.n)
    b[0] = 1.0
    for mode in ("async", "sync-block"):
        x, info = _solve(bar, A, b, 128, 5, mode, 20000, 1e-13)
        assert info["converged"] and abs(x[0] - ref) < 1e-11


# ------------------------------------------------------------------ every kernel generation
@pytest.mark.parametrize("tune", [{"kernel": "block"}, {"kernel": "reg"}, {"kernel": "reg_tma"}, {"kernel": "pers"},
                                  {"pipe": 1}, {"pipe": -1}, {"jacobi_rowwise": 1}, {"single_launch": 1},
                                  {"single_launch": -1}, {"ghost_prefetch": -1}, {"ghost_prefetch": 1},
                                  {"async_queue": "queue"}, {"resident": -1}, {"lead": 3}, {"graph": -1},
                                  {"lazy_publish": 1}, {"lazy_publish": 2}, {"lazy_publish": -1},
                                  {"gather_ahead": -1}, {"fuse_residual": -1}])
@pytest.mark.parametrize("name,R", [("fv1", 128), ("s7_m12", 288), ("tref2000", 128), ("s7_m12", 512),
                                    ("rand", 1024)])
def test_forced_kernel_paths(bar, tune, name, R):
    """Each kernel the dispatcher can choose (fallbacks included, forced through the handle's
    bar_tuning; for the single-launch kernel each residual-publication scheme, the gathers at the
    sweep's start and the separate confirming residual) gives the oracle's iterates in the sync
    modes and converges in async."""
    A = MATS[name]()
    b = np.ones(A.n)
    x0 = np.random.default_rng(2).uniform(-1, 1, A.n)
    for mode, k in (("sync-block", 5), ("jacobi", 1)):
        ref = x0
        for _ in range(3):
            ref = O.jacobi_step(A, b, ref) if mode == "jacobi" else O.block_jacobi_step(A, b, ref, R, k)
        x, _ = _solve(bar, A, b, R, k, mode, 3, 0.0, x0, tuning=tune)
        _close(x, ref)
    x, info = _solve(bar, A, b, R, 5, "async", 20000, 1e-10, tuning=tune)
    assert info["converged"] and O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)


def test_tuning_validation(bar):
    A = W.trefethen(64)
    M = bar.Matrix.from_csr(A, 16)
    for bad in ({"kernel": 9}, {"lead": 49}, {"async_order": 4}, {"halo": 2}, {"warps": 33}, {"peer": 1}):
        with pytest.raises(bar.BarError):
            M.set_tuning(bad)
    with pytest.raises(KeyError):
        bar.Tuning.make(no_such_field=1)
    M.set_tuning(None)
    M.close()


# ------------------------------------------------------------------ pipelined / two-blocks-per-SM
@pytest.mark.parametrize("tune", [{"duo": 1}, {"duo": -1}, {"duo": -1, "pipe": -1}, {"duo": 1, "coded": -1},
                                  {"duo": 1, "coded": 2}, {"async_order": "round_robin"}, {"async_order": "chunks"},
                                  {"async_order": "fronts", "fronts": 4}])
def test_large_subdomain_kernels(bar, tune):
    """C5's shape at a testable size: 3D 7-point, m = 128, R = 256 = two grid lines (so a row has
    at most 4 local entries, as at 512^3 with R = 1024). The two-blocks-per-SM kernel
    (k_block_duo), the pipelined kernel (k_block_pipe) and the one-ahead kernel (k_block_stage)
    give the oracle's sync-block-(5) and Jacobi iterates and converge in async."""
    A = W.stencil7_3d(128)
    R = 256
    b = np.ones(A.n)
    x0 = np.random.default_rng(5).uniform(-1, 1, A.n)
    for mode, k in (("sync-block", 5), ("jacobi", 1)):
        ref = x0
        for _ in range(2):
            ref = O.jacobi_step(A, b, ref) if mode == "jacobi" else O.block_jacobi_step(A, b, ref, R, k)
        x, _ = _solve(bar, A, b, R, k, mode, 2, 0.0, x0, tuning=tune)
        _close(x, ref)
    x, info = _solve(bar, A, b, R, 5, "async", 20000, 1e-10, tuning=tune)
    assert info["converged"] and O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)


def test_coded_columns(bar):
    """Coded columns (1-byte codes into per-subdomain offset dictionaries) are built for stencils
    and give bitwise the int32-column iterates; matrices with more than 256 distinct column offsets
    in a subdomain keep the int32 columns only (and still match the oracle)."""
    A = W.stencil7_3d(128)  # R = two grid lines: <= 4 local entries per row, the duo kernel applies
    R = 256
    M = bar.Matrix.from_csr(A, R)
    assert M.info()["coded"] == 1
    assert M.info()["layout_bytes_per_iter"] < M.info()["model_bytes_per_iter"]
    b = _dev(np.ones(A.n))
    x0 = _dev(np.random.default_rng(9).uniform(-1, 1, A.n))
    out = {}
    names = {2: "staged", 1: "coded", 0: "coded", -1: None}
    for coded in (2, 1, 0, -1):  # the sync modes pick the duo kernel only for larger slabs: force it
        M.set_tuning(duo=1, coded=coded)
        for mode, k in (("sync-block", 5), ("jacobi", 1)):
            x, info = M.solve(b, x0, k=k, max_global_iters=4, tol=0.0, mode=mode)
            out[coded, mode] = x.cpu().numpy()
            kern = M.info()["last_sweep_kernel"]
            assert (names[coded] in kern) if names[coded] else ("," not in kern), (coded, kern)
    for mode in ("sync-block", "jacobi"):  # staged gathers, coded columns, int32 columns: the same bits
        assert np.array_equal(out[1, mode], out[-1, mode])
        assert np.array_equal(out[0, mode], out[-1, mode])
        assert np.array_equal(out[2, mode], out[-1, mode])
    R = W.random_dd(4096, nnz_per_row=7, seed=3)
    MR = bar.Matrix.from_csr(R, 1024)
    assert MR.info()["coded"] == 0


def test_concurrent_handles_threads(bar):
    """Two matrices solved at the same time from two host threads on two streams (the launchers'
    static caches are shared): both results meet the exact residual."""
    import threading

    import torch

    mats = [W.trefethen(2000), W.stencil9_2d(98)]
    out = [None, None]

    def work(t):
        A = mats[t]
        st = torch.cuda.Stream()
        M = bar.Matrix.from_csr(A, 128)
        b = _dev(np.ones(A.n))
        for _ in range(20):
            with torch.cuda.stream(st):
                x, info = M.solve(b, None, None, k=5, tol=1e-10, mode="async", stream=st)
        st.synchronize()
        out[t] = (x.cpu().numpy(), info)
        M.close()

    ths = [threading.Thread(target=work, args=(t,)) for t in range(2)]
    for th in ths:
        th.start()
    for th in ths:
        th.join()
    for t in range(2):
        x, info = out[t]
        assert info["converged"] and O.rel_res(mats[t], np.ones(mats[t].n), x) <= 1e-10 * (1 + 1e-6)


def test_graph_replay(bar):
    """Repeated single-launch solves replay a captured graph: same pointers (new contents of b are
    read), new pointers (recaptured), max_global_iters / tol changes, and tuning.graph = -1 all give
    solutions that meet the exact residual; the graph's kernel time is reported."""
    import torch

    A = W.trefethen(2000)
    M = bar.Matrix.from_csr(A, 128)
    b = _dev(np.ones(A.n))
    x = torch.empty_like(b)
    infos = []
    for rep in range(3):
        _, info = M.solve(b, None, x, k=5, tol=1e-10, mode="async")
        infos.append(info)
        assert info["converged"] and O.rel_res(A, np.ones(A.n), x.cpu().numpy()) <= 1e-10 * (1 + 1e-6)
    assert infos[-1]["sweep_kernel_ms"] > 0 and infos[-1]["sweep_kernel_iters"] > 0
    b2 = np.random.default_rng(4).uniform(0.5, 1.5, A.n)
    b.copy_(torch.from_numpy(b2))  # same pointer, new right-hand side
    _, info = M.solve(b, None, x, k=5, tol=1e-10, mode="async")
    assert info["converged"] and O.rel_res(A, b2, x.cpu().numpy()) <= 1e-10 * (1 + 1e-6)
    x2 = torch.empty_like(b)  # new output pointer: recaptured
    _, info = M.solve(b, None, x2, k=5, tol=1e-12, mode="async")
    assert info["converged"] and O.rel_res(A, b2, x2.cpu().numpy()) <= 1e-12 * (1 + 1e-6)
    _, info = M.solve(b, None, x2, k=5, max_global_iters=3, tol=0.0, mode="async")
    assert info["iters"] == 3 and not info["converged"]
    M.set_tuning(graph=-1)
    _, info = M.solve(b, None, x, k=5, tol=1e-10, mode="async")
    assert info["converged"] and O.rel_res(A, b2, x.cpu().numpy()) <= 1e-10 * (1 + 1e-6)
    M.close()


@pytest.mark.parametrize("coded", [0, 2, -1])
def test_duo_partial_last_subdomain(bar, coded):
    """The two-blocks-per-SM kernel (coded and int32 columns) on a 2D 9-point stencil whose last
    subdomain is partial (n = 10^6 is not a multiple of R = 512, so its last slices are short and
    padded): sync-block-(5) and Jacobi iterates match the oracle to 1e-12, async converges."""
    tune = {"duo": 1, "coded": coded}
    A = W.stencil9_2d(1000)
    R = 512
    b = np.ones(A.n)
    x0 = np.random.default_rng(11).uniform(-1, 1, A.n)
    for mode, k in (("sync-block", 5), ("jacobi", 1)):
        ref = x0
        for _ in range(2):
            ref = O.jacobi_step(A, b, ref) if mode == "jacobi" else O.block_jacobi_step(A, b, ref, R, k)
        x, _ = _solve(bar, A, b, R, k, mode, 2, 0.0, x0, tuning=tune)
        _close(x, ref)
    x, info = _solve(bar, A, b, R, 5, "async", 20000, 1e-10, tuning=tune)
    assert info["converged"] and O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)


@pytest.mark.parametrize("name,gen,R", [("s7_m128", lambda: W.stencil7_3d(128), 256),
                                        ("s9_m600", lambda: W.stencil9_2d(600), 512),
                                        ("s7_m192", lambda: W.stencil7_3d(192), 384)])
def test_staged_gathers(bar, name, gen, R):
    """Staged gathers (k_block_duo<.., staged>, tuning.coded = 2: each subdomain's off-block x
    intervals copied into shared memory once per visit, Layout::iv / sdict) on stencil matrices
    (3D grid planes and lines, 2D subdomains that straddle grid lines with a partial last
    subdomain): sync-block and Jacobi iterates match the oracle to 1e-12, async converges."""
    A = gen()
    b = np.ones(A.n)
    x0 = np.random.default_rng(21).uniform(-1, 1, A.n)
    M = bar.Matrix.from_csr(A, R, tuning={"duo": 1, "coded": 2, "single_launch": -1})
    import torch

    for mode, k in (("sync-block", 5), ("jacobi", 1), ("sync-block", 2)):
        ref = x0
        for m in range(1, 4):
            ref = O.jacobi_step(A, b, ref) if mode == "jacobi" else O.block_jacobi_step(A, b, ref, R, k)
        x = torch.empty(A.n, dtype=torch.float64, device="cuda")
        M.solve(_dev(b), _dev(x0), x, k=k, max_global_iters=3, tol=0.0, mode=mode)
        assert "staged" in M.info()["last_sweep_kernel"], M.info()["last_sweep_kernel"]
        _close(x.cpu().numpy(), ref)
    x, info = M.solve(_dev(b), None, None, k=5, tol=1e-10, mode="async")
    assert "staged" in M.info()["last_sweep_kernel"]
    assert info["converged"] and O.rel_res(A, b, x.cpu().numpy()) <= 1e-10 * (1 + 1e-6)
    M.close()
    # matrices whose off-block columns are not a few intervals keep the entry-by-entry gathers
    Rm = W.random_dd(8192, nnz_per_row=5, seed=9, symmetric_pattern=True)
    MR = bar.Matrix.from_csr(Rm, 512, tuning={"duo": 1, "coded": 2})
    MR.solve(_dev(np.ones(Rm.n)), None, None, k=5, max_global_iters=2, tol=0.0, mode="sync-block")
    assert "staged" not in MR.info()["last_sweep_kernel"]
    MR.close()


@pytest.mark.parametrize("name,gen,R", [("s9_m600", lambda: W.stencil9_2d(600), 512),
                                        ("s7_m128", lambda: W.stencil7_3d(128), 256)])
@pytest.mark.parametrize("stage_bx", [0, -1])
@pytest.mark.parametrize("grid_cap", [0, 5])
@pytest.mark.parametrize("unroll_off", [0, -1])
def test_duo_slab_staging_and_buffer_rotation(bar, name, gen, R, stage_bx, grid_cap, unroll_off):
    """k_block_duo with b_J / x_J bulk-copied with the slab (tuning.stage_bx = 0, the default
    where the blocks per SM stay the same) and with per-row loads (-1); grid_cap = 5
    makes every block sweep dozens of subdomains in a row, which exercises the y-buffer rotation
    that replaces the end-of-subdomain barrier (k odd: buffers swap, k even: no swap, k = 1:
    barrier). unroll_off: the unrolled phase 1 (0; wo4 on the 3D stencil's <= 4 off-block entries
    per row; the 2D stencil's up to 7 keep the generic loop) and the generic loop (-1). Sync-block-(k) for k = 2, 3, 5 and Jacobi match the oracle to
    1e-12 after 3 iterations; async-(5) converges."""
    import torch

    A = gen()
    b = np.random.default_rng(5).uniform(0.5, 1.5, A.n)
    x0 = np.random.default_rng(6).uniform(-1, 1, A.n)
    M = bar.Matrix.from_csr(A, R, tuning={"duo": 1, "single_launch": -1, "stage_bx": stage_bx,
                                          "grid_cap": grid_cap, "unroll_off": unroll_off})
    kernels = set()
    for mode, k in (("sync-block", 5), ("sync-block", 2), ("sync-block", 3), ("jacobi", 1)):
        ref = x0
        for _ in range(3):
            ref = O.jacobi_step(A, b, ref) if mode == "jacobi" else O.block_jacobi_step(A, b, ref, R, k)
        x = torch.empty(A.n, dtype=torch.float64, device="cuda")
        M.solve(_dev(b), _dev(x0), x, k=k, max_global_iters=3, tol=0.0, mode=mode)
        kernels.add(M.info()["last_sweep_kernel"])
        _close(x.cpu().numpy(), ref)
    x, info = M.solve(_dev(b), None, None, k=5, tol=1e-10, mode="async")
    kernels.add(M.info()["last_sweep_kernel"])
    assert info["converged"] and O.rel_res(A, b, x.cpu().numpy()) <= 1e-10 * (1 + 1e-6)
    M.close()
    assert all(kn.startswith("k_block_duo<") and ",coded" in kn for kn in kernels), kernels
    want = ",wo4" if unroll_off == 0 and name == "s7_m128" else None
    assert all((",wo" not in kn) if want is None else (want + "," in kn or want + ">" in kn) for kn in kernels), kernels
    staged = {kn for kn in kernels if kn.endswith(",bx>")}
    if stage_bx < 0:
        assert not staged, kernels
    elif name == "s7_m128":  # C5's geometry (R = two grid lines): the staged variant keeps two blocks per SM
        assert staged, kernels


def _banded_random(n, band, per_row, seed):
    """Seeded banded random matrix: per row the diagonal plus `per_row` distinct offsets in
    [-band, band] (clipped at the matrix edges), off-diagonals uniform in [-1, -0.1], diagonal
    1.5 x the row's absolute off-diagonal sum (rho(|B|) <= 2/3). Few distinct column offsets per
    subdomain (coded columns) with random values and a ragged pattern near the subdomain edges."""
    rng = np.random.default_rng(seed)
    offs = np.array([d for d in range(-band, band + 1) if d != 0])
    pick = np.argsort(rng.random((n, offs.size)), axis=1)[:, :per_row]
    d = np.sort(offs[pick], axis=1)
    rows = np.arange(n)[:, None]
    c = rows + d
    ok = (c >= 0) & (c < n)
    v = -rng.uniform(0.1, 1.0, size=d.shape)
    v[~ok] = 0.0
    diag = 1.5 * np.abs(v).sum(axis=1) + 1.0
    cols = np.concatenate([np.where(ok, c, -1), rows], axis=1)
    vals = np.concatenate([v, diag[:, None]], axis=1)
    order = np.argsort(cols, axis=1, kind="stable")
    cols = np.take_along_axis(cols, order, axis=1)
    vals = np.take_along_axis(vals, order, axis=1)
    keep = cols >= 0
    counts = keep.sum(axis=1)
    rowptr = np.zeros(n + 1, dtype=np.int32)
    rowptr[1:] = np.cumsum(counts)
    return W.CSR(n, rowptr, cols[keep].astype(np.int32), vals[keep].astype(np.float64), name=f"banded_{n}_{seed}")


@pytest.mark.parametrize("n,R,seed", [(1_000_123, 256, 1), (1_000_123, 512, 2), (700_001, 1024, 3)])
@pytest.mark.parametrize("unroll_off", [0, -1])
def test_duo_unrolled_random_banded(bar, n, R, seed, unroll_off):
    """The two-blocks-per-SM kernel's unrolled phase 1 (<= 4 off-block entries per row, coded
    columns; `wo4` in the kernel name) against the generic loop (-1) on random banded matrices:
    random values (not a stencil's constant coefficients), rows with 0-3 off-block entries in any
    position, a partial last subdomain and partial last slice (n not a multiple of R or 32).
    Sync-block-(k) for k = 1, 3, 5 and Jacobi match the oracle to 1e-12 after 2 iterations;
    async-(5) meets the exact residual."""
    import torch

    A = _banded_random(n, 60, 3, seed)  # <= 4 local entries (the duo kernel), <= 3 off-block
    b = np.random.default_rng(seed + 100).uniform(0.5, 1.5, n)
    x0 = np.random.default_rng(seed + 200).uniform(-1, 1, n)
    M = bar.Matrix.from_csr(A, R, tuning={"duo": 1, "single_launch": -1, "unroll_off": unroll_off})
    assert M.info()["coded"] == 1
    kernels = set()
    for mode, k in (("sync-block", 5), ("sync-block", 3), ("sync-block", 1), ("jacobi", 1)):
        ref = x0
        for _ in range(2):
            ref = O.jacobi_step(A, b, ref) if mode == "jacobi" else O.block_jacobi_step(A, b, ref, R, k)
        x = torch.empty(n, dtype=torch.float64, device="cuda")
        M.solve(_dev(b), _dev(x0), x, k=k, max_global_iters=2, tol=0.0, mode=mode)
        kernels.add(M.info()["last_sweep_kernel"])
        _close(x.cpu().numpy(), ref)
    x, info = M.solve(_dev(b), None, None, k=5, tol=1e-10, mode="async")
    kernels.add(M.info()["last_sweep_kernel"])
    assert info["converged"] and O.rel_res(A, b, x.cpu().numpy()) <= 1e-10 * (1 + 1e-6)
    M.close()
    assert all(kn.startswith("k_block_duo<") for kn in kernels), kernels
    assert all((",wo4" in kn) == (unroll_off == 0) for kn in kernels), kernels

"""GPU parity of bar_solve_ex's options against the oracle:
N3 tau-scaled relaxation, N1 failure injection (§4.5), residual history."""
import numpy as np
import pytest

import oracle as O
import workloads as W

pytestmark = pytest.mark.gpu


def _dev(a):
    import torch

    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def _gpu(bar, A, b, R, k, mode, iters, tol, x0=None, tuning=None, **kw):
    M = bar.Matrix.from_csr(A, R, tuning=tuning)
    x, info = M.solve(_dev(b), None if x0 is None else _dev(x0), None, k=k, max_global_iters=iters, tol=tol,
                      mode=mode, **kw)
    M.close()
    return x.cpu().numpy(), info


def _close(x, ref, tol=1e-12):
    assert np.abs(x - ref).max() <= tol * np.abs(ref).max(), np.abs(x - ref).max()


MATS = {"tref2000": (lambda: W.trefethen(2000), 128), "fv1": (lambda: W.stencil9_2d(98), 128),
        "s7": (lambda: W.stencil7_3d(16), 1024), "rand": (lambda: W.random_dd(1500, 6, seed=4), 100)}


@pytest.mark.parametrize("name", list(MATS))
@pytest.mark.parametrize("mode,k", [("sync-block", 5), ("jacobi", 1), ("sync-block", 2)])
@pytest.mark.parametrize("tau", [0.7, 1.15])
def test_tau_iterates(bar, name, mode, k, tau):
    gen, R = MATS[name]
    A = gen()
    b = np.ones(A.n)
    x0 = np.random.default_rng(9).uniform(-1, 1, A.n)
    meth = O.JACOBI if mode == "jacobi" else O.BLOCK_JACOBI
    ref = x0
    for m in range(1, 7):
        ref = O.step_ex(A, b, ref, meth, R=R, k=k, tau=tau)
        if m in (1, 6):
            x, info = _gpu(bar, A, b, R, k, mode, m, 0.0, x0, tau=tau)
            _close(x, ref)


def test_tau_rho_gt_1(bar):
    """SPD with rho(B) > 1: Jacobi diverges, tau = 2/(lambda_1 + lambda_n) converges."""
    n = 48
    Ad = np.eye(n) + 0.3 * np.ones((n, n))  # SPD, rho(B) = 0.3 (n-1) / 1.3 > 1
    nz = [np.nonzero(Ad[i])[0] for i in range(n)]
    A = W.CSR(n, np.concatenate([[0], np.cumsum([len(z) for z in nz])]).astype(np.int32),
              np.concatenate(nz).astype(np.int32), np.concatenate([Ad[i, z] for i, z in enumerate(nz)]))
    DA = Ad / np.diag(Ad)[:, None]
    lam = np.linalg.eigvals(DA).real
    if np.abs(np.linalg.eigvals(np.eye(n) - DA)).max() <= 1:
        pytest.skip("generated matrix has rho(B) <= 1")
    tau = 2.0 / (lam.min() + lam.max())
    b = np.ones(n)
    _, info = _gpu(bar, A, b, 64, 1, "jacobi", 5000, 1e-10, raise_on_error=False)
    assert info["status"] == "BAR_ERR_DIVERGED"
    x, info = _gpu(bar, A, b, 64, 1, "jacobi", 5000, 1e-10, tau=tau)
    r = O.solve(A, b, method=O.JACOBI, tol=1e-10, max_iters=5000, tau=tau)
    assert info["converged"] and info["iters"] == r.iters
    _close(x, r.x, 1e-10)


def test_tau_async(bar):
    """N3 in async mode (§8(f): "all three modes").
    * The SPD system with rho(B) > 1: with tau = 2/(lambda_1 + lambda_n) async-(1)
      converges to the direct solution. Across several subdomains nothing guarantees that
      (rho(|B_tau|) = 1 - tau + tau rho(|B|) > 1 for every tau <= 1, so Chazan-Miranker allows
      divergent orders), so it runs on one subdomain (R >= n), where async-(1) is tau-Jacobi.
    * With tau != 1 the fixed point is preserved (start at x*, tol = 0: x stays at x*), and
      for tau < 1 on Trefethen_2000 (rho(|B_tau|) = 1 - tau + 0.86 tau < 1) async-(5) over 16
      subdomains converges to x*."""
    n = 48
    Ad = np.eye(n) + 0.3 * np.ones((n, n))
    nz = [np.nonzero(Ad[i])[0] for i in range(n)]
    A = W.CSR(n, np.concatenate([[0], np.cumsum([len(z) for z in nz])]).astype(np.int32),
              np.concatenate(nz).astype(np.int32), np.concatenate([Ad[i, z] for i, z in enumerate(nz)]))
    DA = Ad / np.diag(Ad)[:, None]
    lam = np.linalg.eigvals(DA).real
    tau = 2.0 / (lam.min() + lam.max())
    b = np.ones(n)
    xs = np.linalg.solve(Ad, b)
    for R in (64, 1024):
        x, info = _gpu(bar, A, b, R, 1, "async", 20000, 1e-10, tau=tau)
        assert info["converged"] and O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)
        _close(x, xs, 1e-8)
    B = W.trefethen(2000)
    bb = np.ones(B.n)
    xb = np.linalg.solve(B.to_dense(), bb)
    for tau_ in (0.7, 1.2):
        x, info = _gpu(bar, B, bb, 128, 5, "async", 10, 0.0, xb, tau=tau_)
        assert info["iters"] == 10
        assert np.abs(x - xb).max() <= 1e-13 * np.abs(xb).max()
        # and from x0 = 0 the tau-scaled async iteration converges (rho(|B_tau|) < 1 for tau <= 1)
        if tau_ < 1:
            x, info = _gpu(bar, B, bb, 128, 5, "async", 20000, 1e-10, tau=tau_)
            assert info["converged"] and np.abs(x - xb).max() <= 1e-8 * np.abs(xb).max()


@pytest.mark.parametrize("name", list(MATS))
@pytest.mark.parametrize("mode,k", [("sync-block", 5), ("jacobi", 1)])
def test_failure_window_iterates(bar, name, mode, k):
    """25% of the components frozen in global iterations 3..6: iterate-by-iterate parity and the
    same stopping iteration as the oracle's masked solve."""
    gen, R = MATS[name]
    A = gen()
    b = np.ones(A.n)
    fz = (np.random.default_rng(3).random(A.n) < 0.25).astype(np.uint8)
    meth = O.JACOBI if mode == "jacobi" else O.BLOCK_JACOBI
    for m in (2, 4, 8):
        r = O.solve(A, b, method=meth, R=R, k=k, tol=0.0, max_iters=m, frozen=fz, fail_start=3, fail_stop=7)
        x, info = _gpu(bar, A, b, R, k, mode, m, 0.0, fail_mask=fz, fail_start=3, fail_stop=7)
        _close(x, r.x)
    r = O.solve(A, b, method=meth, R=R, k=k, tol=1e-10, frozen=fz, fail_start=3, fail_stop=7)
    x, info = _gpu(bar, A, b, R, k, mode, 20000, 1e-10, fail_mask=fz, fail_start=3, fail_stop=7)
    assert info["converged"] and info["iters"] == r.iters
    _close(x, r.x)


def test_failure_never_recovers_async(bar):
    """Without recovery the frozen components never move (async-(5)); with recovery async
    converges, later than without failures (§4.5, Fig. 10)."""
    A = W.trefethen(2000)
    b = np.ones(A.n)
    fz = (np.random.default_rng(6).random(A.n) < 0.25).astype(np.uint8)
    x, info = _gpu(bar, A, b, 128, 5, "async", 60, 1e-10, fail_mask=fz, fail_start=1, fail_stop=-1)
    assert not info["converged"] and np.all(x[fz == 1] == 0.0)
    _, base = _gpu(bar, A, b, 128, 5, "async", 20000, 1e-10)
    x, info = _gpu(bar, A, b, 128, 5, "async", 20000, 1e-10, fail_mask=fz, fail_start=10, fail_stop=30)
    assert info["converged"] and info["iters"] > base["iters"]
    assert O.rel_res(A, b, x) <= 1e-10 * (1 + 1e-6)


@pytest.mark.parametrize("mode,k", [("sync-block", 5), ("jacobi", 1)])
def test_history_matches_oracle(bar, mode, k):
    A = W.stencil9_2d(98)
    b = np.ones(A.n)
    meth = O.JACOBI if mode == "jacobi" else O.BLOCK_JACOBI
    r = O.solve(A, b, method=meth, R=128, k=k, tol=1e-10)
    _, info = _gpu(bar, A, b, 128, k, mode, 20000, 1e-10, history=True)
    h = info["history"]
    assert len(h) == r.iters + 1
    np.testing.assert_allclose(h, r.history, rtol=1e-9, atol=1e-15)


@pytest.mark.parametrize("coded", [0, 2, -1])
def test_ext_options_on_duo_kernel(bar, coded):
    """N3 tau-scaling and N1 failure windows through the two-blocks-per-SM kernel's EXT
    instantiations (coded and int32 columns): iterates match the oracle to 1e-12."""
    tune = {"duo": 1, "coded": coded}
    A = W.stencil7_3d(128)  # R = two grid lines: <= 4 local entries per row
    R = 256
    b = np.ones(A.n)
    x0 = np.random.default_rng(13).uniform(-1, 1, A.n)
    for mode, k, meth in (("sync-block", 5, O.BLOCK_JACOBI), ("jacobi", 1, O.JACOBI)):
        ref = x0
        for _ in range(2):
            ref = O.step_ex(A, b, ref, meth, R=R, k=k, tau=0.8)
        x, _ = _gpu(bar, A, b, R, k, mode, 2, 0.0, x0, tuning=tune, tau=0.8)
        _close(x, ref)
    fz = np.random.default_rng(14).random(A.n) < 0.25
    r = O.solve(A, b, method=O.BLOCK_JACOBI, R=R, k=5, tol=0.0, max_iters=4, frozen=fz, fail_start=2, fail_stop=4)
    x, _ = _gpu(bar, A, b, R, 5, "sync-block", 4, 0.0, tuning=tune, fail_mask=fz, fail_start=2, fail_stop=4)
    _close(x, r.x)


def test_n2_harness_small(bar):
    """tools/nondeterminism.py (N2, Tables 2-3) at a small size: every run of a fixed
    iteration count returns a finite exact residual, residuals fall with m, and the spread is
    reported (run-to-run variation of the asynchronous schedule)."""
    from tools import nondeterminism

    name, rows = nondeterminism.table("c1", runs=4, checkpoints=[5, 15, 25])
    assert [m for m, _ in rows] == [5, 15, 25]
    avgs = [r.mean() for _, r in rows]
    for _, r in rows:
        assert len(r) == 4 and np.all(np.isfinite(r)) and np.all(r > 0)
    assert avgs[0] > avgs[1] > avgs[2]
    # sync-block-(5) after m iterations bounds the async average within a factor 30 (P5, R15)
    A = W.trefethen(2000)
    for m, r in rows:
        sb = O.solve(A, np.ones(A.n), method=O.BLOCK_JACOBI, R=128, k=5, tol=0.0, max_iters=m).rel_res
        assert r.mean() <= 30 * sb, (m, r.mean(), sb)


def test_n4_harness_small(bar):
    """tools/local_iters.py (N4, Table 4, P:711 / P:863-867) on C2: positive per-iteration times
    for k = 1, 5, 9 that do not fall with k (each extra local sweep adds work, no HBM bytes)."""
    from tools import local_iters

    info, kernel, rows = local_iters.table("c2", ks=(1, 5, 9))
    ts = [t for _, t in rows]
    assert all(t > 0 for t in ts), rows
    assert ts[2] >= 0.9 * ts[0], rows

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


def _gpu(bar, A, b, R, k, mode, iters, tol, x0=None, **kw):
    M = bar.Matrix.from_csr(A, R)
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


@pytest.mark.parametrize("coded", ["1", "0"])
def test_ext_options_on_duo_kernel(bar, monkeypatch, coded):
    """N3 tau-scaling and N1 failure windows through the two-blocks-per-SM kernel's EXT
    instantiations (coded and int32 columns): iterates match the oracle to 1e-12."""
    monkeypatch.setenv("BAR_DUO", "1")
    monkeypatch.setenv("BAR_CODED", coded)
    A = W.stencil7_3d(128)  # R = two grid lines: <= 4 local entries per row
    R = 256
    b = np.ones(A.n)
    x0 = np.random.default_rng(13).uniform(-1, 1, A.n)
    for mode, k, meth in (("sync-block", 5, O.BLOCK_JACOBI), ("jacobi", 1, O.JACOBI)):
        ref = x0
        for _ in range(2):
            ref = O.step_ex(A, b, ref, meth, R=R, k=k, tau=0.8)
        x, _ = _gpu(bar, A, b, R, k, mode, 2, 0.0, x0, tau=0.8)
        _close(x, ref)
    fz = np.random.default_rng(14).random(A.n) < 0.25
    r = O.solve(A, b, method=O.BLOCK_JACOBI, R=R, k=5, tol=0.0, max_iters=4, frozen=fz, fail_start=2, fail_stop=4)
    x, _ = _gpu(bar, A, b, R, 5, "sync-block", 4, 0.0, fail_mask=fz, fail_start=2, fail_stop=4)
    _close(x, r.x)

"""Generator pins: PAPER.md Table 1 and closed forms."""
import numpy as np
import pytest

import workloads as W


def _table1(golden):
    return {r[0]: r[1:] for r in golden("table1.txt")}


@pytest.mark.parametrize("n,last_prime,minlen,maxlen", [(2000, 17389, 12, 22), (20000, 224737, 16, 29)])
def test_trefethen_table1(golden, n, last_prime, minlen, maxlen):
    t1 = _table1(golden)
    A = W.trefethen(n)
    assert A.n == int(t1[f"Trefethen_{n}"][0])
    assert A.nnz == int(t1[f"Trefethen_{n}"][1])          # 41,906 / 554,466
    # closed form nnz = n + 2 * sum_{2^t < n} (n - 2^t)
    cf = n + 2 * sum(n - (1 << t) for t in range(64) if (1 << t) < n)
    assert A.nnz == cf
    d = A.val[[A.rowptr[i] + np.searchsorted(A.col[A.rowptr[i]:A.rowptr[i + 1]], i) for i in (0, 1, n - 1)]]
    assert d.tolist() == [2.0, 3.0, float(last_prime)]
    lens = np.diff(A.rowptr)
    assert lens.min() == minlen and lens.max() == maxlen


def test_trefethen_structure_bruteforce():
    """Tiny n against a brute-force dense definition (primes by trial division)."""
    n = 37
    primes = [p for p in range(2, 1000) if all(p % q for q in range(2, int(p ** 0.5) + 1))][:n]
    dense = np.diag(np.array(primes, dtype=float))
    for i in range(n):
        for j in range(n):
            dd = abs(i - j)
            if dd and (dd & (dd - 1)) == 0:
                dense[i, j] = 1.0
    np.testing.assert_array_equal(W.trefethen(n).to_dense(), dense)


def test_trefethen_spectral_table1(golden):
    """rho(B) = 0.8601 and cond_1(D^-1 A) = 6.1579 for Trefethen_2000 (Table 1)."""
    t1 = _table1(golden)
    A = W.trefethen(2000).to_dense()
    d = np.diag(A)
    B = np.eye(2000) - A / d[:, None]
    rho = np.abs(np.linalg.eigvals(B)).max()
    assert round(rho, 4) == float(t1["Trefethen_2000"][4])
    rho_abs = np.abs(np.linalg.eigvals(np.abs(B))).max()
    assert round(rho_abs, 4) == float(t1["Trefethen_2000"][4])
    DA = A / d[:, None]
    assert round(np.linalg.cond(DA, 1), 4) == float(t1["Trefethen_2000"][3])


@pytest.mark.parametrize("m,name", [(98, "fv1"), (99, "fv2")])
def test_stencil9_pattern_matches_fv(golden, m, name):
    """The fv1/fv2/fv3 pattern: 9-point stencil, nnz = (3m-2)^2 (Table 1)."""
    t1 = _table1(golden)
    A = W.stencil9_2d(m)
    assert A.n == int(t1[name][0]) and A.nnz == int(t1[name][1]) == (3 * m - 2) ** 2


def test_stencil9_rho_closed_form(golden):
    """rho(B) = ((1+2cos(pi/(m+1)))^2 - 1)/d; d = 9.3595 gives fv1's 0.8541 (Table 1)."""
    t1 = _table1(golden)
    m, d = 98, W.FV1_DIAG
    cf = ((1 + 2 * np.cos(np.pi / (m + 1))) ** 2 - 1) / d
    assert round(cf, 4) == float(t1["fv1"][4])
    # the generated matrix has exactly this spectrum: A = (d+1) I - T (x) T, T = tridiag(1,1,1)
    ms = 12
    A = W.stencil9_2d(ms, d).to_dense()
    T = np.eye(ms) + np.eye(ms, k=1) + np.eye(ms, k=-1)
    np.testing.assert_array_equal(A, (d + 1) * np.eye(ms * ms) - np.kron(T, T))
    B = np.eye(ms * ms) - A / d
    rho = np.abs(np.linalg.eigvalsh(B)).max()
    assert abs(rho - ((1 + 2 * np.cos(np.pi / (ms + 1))) ** 2 - 1) / d) < 1e-12


def test_stencil7_closed_forms():
    m = 9
    A = W.stencil7_3d(m)
    assert A.nnz == 7 * m ** 3 - 6 * m ** 2
    D = A.to_dense()
    np.testing.assert_array_equal(D, D.T)
    B = np.eye(m ** 3) - D / W.S7_DIAG
    rho = np.abs(np.linalg.eigvalsh(B)).max()
    assert abs(rho - 6 * np.cos(np.pi / (m + 1)) / W.S7_DIAG) < 1e-12
    # the C5 size fits int32 row pointers: 7*512^3 - 6*512^2 < 2^31
    assert 7 * 512 ** 3 - 6 * 512 ** 2 == 937_951_232 < 2 ** 31


@pytest.mark.parametrize("gen,args,n", [(W.trefethen, (300,), 300), (W.stencil9_2d, (17,), 289),
                                         (W.stencil7_3d, (7,), 343)])
def test_row_ranges_match_full(gen, args, n):
    full = gen(*args)
    for lo, hi in [(0, 1), (5, 77), (n - 13, n), (40, 40)]:
        part = gen(*args, row_lo=lo, row_hi=hi)
        s, e = full.rowptr[lo], full.rowptr[hi]
        np.testing.assert_array_equal(part.rowptr, full.rowptr[lo:hi + 1] - s)
        np.testing.assert_array_equal(part.col, full.col[s:e])
        np.testing.assert_array_equal(part.val, full.val[s:e])


def test_csr_invariants_random_dd():
    for seed in range(5):
        A = W.random_dd(60, 4, seed=seed, symmetric_pattern=bool(seed % 2))
        for i in range(A.n):
            c = A.col[A.rowptr[i]:A.rowptr[i + 1]]
            assert np.all(np.diff(c) > 0) and i in c
        D = A.to_dense()
        B = np.eye(A.n) - D / np.diag(D)[:, None]
        assert np.abs(np.linalg.eigvals(np.abs(B))).max() < 1.0

/*
 * oracle/oracle.c — TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously correct, single-threaded CPU implementation of what
 * the block-asynchronous relaxation paper defines (Anzt, Tomov, Dongarra,
 * Heuveline; /root/reference/PAPER.md, cited as P:<line>). Only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
 * load this library. It shares no code, header or constant with the CUDA path
 * (paper_conf_ipps_anzttdh12_b200/csrc/), and the CUDA path never calls it.
 *
 * Arithmetic: IEEE fp64, compiled with -ffp-contract=off and no fast-math, so
 * every multiply and subtract is rounded separately. Inner sums run in
 * ascending CSR order; the diagonal is applied by DIVISION by a_ii (the
 * component form of eq. 2), never by a multiply with a reciprocal.
 *
 * Functions and the passages they follow:
 *   oracle_jacobi_step        O1  eq. 2: x_i^{m+1} = (b_i - sum_{j!=i} a_ij x_j^m) / a_ii
 *   oracle_block_jacobi_step  O2  Alg. 1, P:147 ("x values used from outside the
 *                                 block are kept constant"), eq. 4 with the
 *                                 DESIGN.md readings R3/R4/R5: per subdomain J_l,
 *                                 s_i = b_i - sum_{j notin J_l} a_ij x_j^m, y^0 = x^m_{J_l},
 *                                 k Jacobi sweeps y_i^{t+1} = (s_i - sum_{j in J_l, j!=i} a_ij y_j^t)/a_ii,
 *                                 x^{m+1}_{J_l} = y^k.
 *   oracle_block_jacobi_subdomain  one subdomain of O2 (for sampled checks at full size).
 *   oracle_gauss_seidel_step  O3  forward Gauss-Seidel, in place, natural order.
 *   oracle_residual_norm      O4  ||b - A x||_2 ("residuals ... always in the l2-norm").
 *   oracle_*_step_ex / oracle_solve_ex  N1 failure injection (§4.5: frozen components)
 *                                 and N3 tau-scaled relaxation (B = I - tau D^-1 A),
 *                                 DESIGN.md readings R17/R18.
 *   oracle_solve              O5  stopping rule of DESIGN.md reading R2/R6: check x^0, then
 *                                 return the first x^m with ||b-Ax^m||/||b|| <= tol, else
 *                                 x^{max_iters} with converged = 0; divergence => status 2.
 *
 * Pins (tests/test_oracle.py): dense LU (numpy dgesv), the fixed-point invariant,
 * closed-form spectral radii and Table 1 values, special-case reductions (k=1, R=1,
 * R>=n), exact dyadic arithmetic, the SIAM (A^-1)_11 constant for Trefethen_20000,
 * brute-force tiny cases, and the paper's Tables 2-3 residual histories (soft pins).
 */
#include <math.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---------------------------------------------------------------- O4 ---- */
/* ||b - A x||_2 over rows [0, nrows) of a CSR block (global column ids).     */
double oracle_residual_norm(int64_t nrows, const int32_t *rowptr, const int32_t *col,
                            const double *val, const double *b, const double *x) {
    double ss = 0.0;
    for (int64_t i = 0; i < nrows; ++i) {
        double r = b[i];
        for (int32_t e = rowptr[i]; e < rowptr[i + 1]; ++e) {
            double t = val[e] * x[col[e]];
            r = r - t;
        }
        double r2 = r * r;
        ss = ss + r2;
    }
    return sqrt(ss);
}

double oracle_norm2(int64_t n, const double *v) {
    double ss = 0.0;
    for (int64_t i = 0; i < n; ++i) {
        double t = v[i] * v[i];
        ss = ss + t;
    }
    return sqrt(ss);
}

/* ---------------------------------------------------------------- O1 ---- */
/* Jacobi (eq. 2) for rows [0, nrows) of a CSR block whose first row is global  */
/* row `row0`: x_new[i] = (b[i] - sum_{j != row0+i} a_ij x_old[j]) / a_ii.       */
int oracle_jacobi_rows(int64_t row0, int64_t nrows, const int32_t *rowptr, const int32_t *col,
                       const double *val, const double *b, const double *x_old, double *x_new) {
    for (int64_t i = 0; i < nrows; ++i) {
        int64_t gi = row0 + i;
        double acc = b[i];
        double aii = 0.0;
        for (int32_t e = rowptr[i]; e < rowptr[i + 1]; ++e) {
            if (col[e] == gi) { aii = val[e]; continue; }
            double t = val[e] * x_old[col[e]];
            acc = acc - t;
        }
        if (aii == 0.0) return -1;
        x_new[i] = acc / aii;
    }
    return 0;
}

int oracle_jacobi_step(int64_t n, const int32_t *rowptr, const int32_t *col, const double *val,
                       const double *b, const double *x_old, double *x_new) {
    return oracle_jacobi_rows(0, n, rowptr, col, val, b, x_old, x_new);
}

/* ---------------------------------------------------------------- O2 ---- */
/* One subdomain J = [TS, TE) of sync-block-(k) (Alg. 1 / eq. 4).               */
/* rowptr/col/val: the CSR rows TS..TE-1 (rowptr relative, global columns).      */
/* b_J: b[TS..TE); x_old: the FULL previous iterate x^m; y_out: TE-TS values.    */
/* work: 2*(TE-TS) doubles of scratch (y^t and s).                               */
int oracle_block_jacobi_subdomain(int64_t TS, int64_t TE, const int32_t *rowptr, const int32_t *col,
                                  const double *val, const double *b_J, const double *x_old,
                                  int32_t k, double *y_out, double *work) {
    int64_t nl = TE - TS;
    double *y = work;          /* y^t */
    double *s = work + nl;     /* off-block part s_i */
    /* Alg. 1 line 2-3: "read x from global memory", s := off-block part. */
    for (int64_t i = 0; i < nl; ++i) {
        double acc = b_J[i];
        for (int32_t e = rowptr[i]; e < rowptr[i + 1]; ++e) {
            int64_t j = col[e];
            if (j >= TS && j < TE) continue;      /* local part handled in the sweeps */
            double t = val[e] * x_old[j];
            acc = acc - t;
        }
        s[i] = acc;
        y[i] = x_old[TS + i];                     /* y^0 = x^m_J */
    }
    /* Alg. 1 lines 4-8: k synchronous Jacobi updates on the subdomain, off-block  */
    /* values frozen; double-buffered (reading R3 in DESIGN.md).            */
    for (int32_t t = 0; t < k; ++t) {
        for (int64_t i = 0; i < nl; ++i) {
            int64_t gi = TS + i;
            double acc = s[i];
            double aii = 0.0;
            for (int32_t e = rowptr[i]; e < rowptr[i + 1]; ++e) {
                int64_t j = col[e];
                if (j < TS || j >= TE) continue;
                if (j == gi) { aii = val[e]; continue; }
                double tt = val[e] * y[j - TS];
                acc = acc - tt;
            }
            if (aii == 0.0) return -1;
            y_out[i] = acc / aii;
        }
        memcpy(y, y_out, sizeof(double) * (size_t)nl);
    }
    if (k == 0) memcpy(y_out, y, sizeof(double) * (size_t)nl);
    return 0;
}

int oracle_block_jacobi_step(int64_t n, const int32_t *rowptr, const int32_t *col, const double *val,
                             const double *b, int64_t R, int32_t k, const double *x_old, double *x_new) {
    if (R < 1 || k < 0) return -2;
    int64_t Rm = R < n ? R : n;
    double *work = (double *)malloc(sizeof(double) * (size_t)(2 * Rm));
    if (!work) return -3;
    int rc = 0;
    for (int64_t TS = 0; TS < n && rc == 0; TS += R) {
        int64_t TE = TS + R < n ? TS + R : n;
        /* rowptr + TS keeps global entry offsets: pass the absolute slice */
        int32_t *rp = (int32_t *)malloc(sizeof(int32_t) * (size_t)(TE - TS + 1));
        if (!rp) { rc = -3; break; }
        for (int64_t i = 0; i <= TE - TS; ++i) rp[i] = rowptr[TS + i] - rowptr[TS];
        rc = oracle_block_jacobi_subdomain(TS, TE, rp, col + rowptr[TS], val + rowptr[TS], b + TS, x_old,
                                           k, x_new + TS, work);
        free(rp);
    }
    free(work);
    return rc;
}

/* ---------------------------------------------------------------- O3 ---- */
/* Forward Gauss-Seidel, in place ("the already computed values of the    */
/* current iteration step are used"; P:139 CPU baseline).                        */
int oracle_gauss_seidel_step(int64_t n, const int32_t *rowptr, const int32_t *col, const double *val,
                             const double *b, double *x) {
    for (int64_t i = 0; i < n; ++i) {
        double acc = b[i];
        double aii = 0.0;
        for (int32_t e = rowptr[i]; e < rowptr[i + 1]; ++e) {
            if (col[e] == i) { aii = val[e]; continue; }
            double t = val[e] * x[col[e]];
            acc = acc - t;
        }
        if (aii == 0.0) return -1;
        x[i] = acc / aii;
    }
    return 0;
}

/* ------------------------------------------- N1 / N3 extensions (oracle) ---- */
/* tau-scaled relaxation (B = I - tau D^-1 A) applied to every update of O1/O2:    */
/*   x_new = x_old + tau * (v - x_old), v the unscaled update; tau == 1 gives v exactly.       */
/* Failure injection (§4.5): components with frozen[i] != 0 keep their value.         */
static double relax(double xold, double v, double tau) { return tau == 1.0 ? v : xold + tau * (v - xold); }

int oracle_jacobi_step_ex(int64_t n, const int32_t *rowptr, const int32_t *col, const double *val,
                          const double *b, const double *x_old, double *x_new, double tau,
                          const uint8_t *frozen) {
    int rc = oracle_jacobi_step(n, rowptr, col, val, b, x_old, x_new);
    if (rc) return rc;
    for (int64_t i = 0; i < n; ++i) {
        if (frozen && frozen[i]) x_new[i] = x_old[i];
        else x_new[i] = relax(x_old[i], x_new[i], tau);
    }
    return 0;
}

int oracle_block_jacobi_step_ex(int64_t n, const int32_t *rowptr, const int32_t *col, const double *val,
                                const double *b, int64_t R, int32_t k, const double *x_old, double *x_new,
                                double tau, const uint8_t *frozen) {
    if (R < 1 || k < 1) return -2;
    for (int64_t TS = 0; TS < n; TS += R) {
        int64_t TE = TS + R < n ? TS + R : n, nl = TE - TS;
        double *y = (double *)malloc(sizeof(double) * (size_t)nl);
        double *yn = (double *)malloc(sizeof(double) * (size_t)nl);
        double *s = (double *)malloc(sizeof(double) * (size_t)nl);
        if (!y || !yn || !s) { free(y); free(yn); free(s); return -3; }
        for (int64_t i = 0; i < nl; ++i) {
            double acc = b[TS + i];
            for (int32_t e = rowptr[TS + i]; e < rowptr[TS + i + 1]; ++e) {
                int64_t j = col[e];
                if (j >= TS && j < TE) continue;
                double t = val[e] * x_old[j];
                acc = acc - t;
            }
            s[i] = acc;
            y[i] = x_old[TS + i];
        }
        for (int32_t t = 0; t < k; ++t) {
            for (int64_t i = 0; i < nl; ++i) {
                int64_t gi = TS + i;
                if (frozen && frozen[gi]) { yn[i] = y[i]; continue; }
                double acc = s[i], aii = 0.0;
                for (int32_t e = rowptr[gi]; e < rowptr[gi + 1]; ++e) {
                    int64_t j = col[e];
                    if (j < TS || j >= TE) continue;
                    if (j == gi) { aii = val[e]; continue; }
                    double tt = val[e] * y[j - TS];
                    acc = acc - tt;
                }
                yn[i] = relax(y[i], acc / aii, tau);
            }
            memcpy(y, yn, sizeof(double) * (size_t)nl);
        }
        memcpy(x_new + TS, y, sizeof(double) * (size_t)nl);
        free(y); free(yn); free(s);
    }
    return 0;
}

/* ---------------------------------------------------------------- O5 ---- */
enum { ORACLE_JACOBI = 0, ORACLE_BLOCK_JACOBI = 1, ORACLE_GAUSS_SEIDEL = 2 };
enum { ORACLE_OK = 0, ORACLE_ERR = 1, ORACLE_DIVERGED = 2 };

/* Solve A x = b from x0 with the chosen relaxation until rel_res <= tol or       */
/* max_iters global iterations. res_hist (nullable) gets rel_res(x^m) for          */
/* m = 0..iters (length >= max_iters + 1).                                          */
/* oracle_solve_ex: O5 with the N1/N3 options: tau-scaling of every update, and components with */
/* frozen[i] != 0 not updated in global iterations m with fail_start <= m < fail_stop            */
/* (fail_stop < 0: never recover). tau = 1, frozen = NULL gives oracle_solve.                    */
int oracle_solve_ex(int32_t method, int64_t n, const int32_t *rowptr, const int32_t *col, const double *val,
                    const double *b, const double *x0, double *x_out, int64_t R, int32_t k,
                    int64_t max_iters, double tol, int64_t *iters_out, double *rel_res_out,
                    int32_t *converged_out, double *res_hist, double tau, const uint8_t *frozen,
                    int64_t fail_start, int64_t fail_stop) {
    double bn = oracle_norm2(n, b);
    *iters_out = 0; *converged_out = 0; *rel_res_out = 0.0;
    if (bn == 0.0) {                       /* b = 0 => x = 0 (reading R2) */
        for (int64_t i = 0; i < n; ++i) x_out[i] = 0.0;
        *converged_out = 1;
        if (res_hist) res_hist[0] = 0.0;
        return ORACLE_OK;
    }
    double *xa = (double *)malloc(sizeof(double) * (size_t)n);
    double *xb = (double *)malloc(sizeof(double) * (size_t)n);
    if (!xa || !xb) { free(xa); free(xb); return ORACLE_ERR; }
    memcpy(xa, x0, sizeof(double) * (size_t)n);
    double rel = oracle_residual_norm(n, rowptr, col, val, b, xa) / bn;
    if (res_hist) res_hist[0] = rel;
    int status = ORACLE_OK;
    int64_t m = 0;
    if (!(rel <= tol)) {
        for (m = 1; m <= max_iters; ++m) {
            int rc = 0;
            const uint8_t *fr = (frozen && m >= fail_start && (fail_stop < 0 || m < fail_stop)) ? frozen : NULL;
            const int plain = tau == 1.0 && fr == NULL;
            if (method == ORACLE_JACOBI) {
                rc = plain ? oracle_jacobi_step(n, rowptr, col, val, b, xa, xb)
                           : oracle_jacobi_step_ex(n, rowptr, col, val, b, xa, xb, tau, fr);
            } else if (method == ORACLE_BLOCK_JACOBI) {
                rc = plain ? oracle_block_jacobi_step(n, rowptr, col, val, b, R, k, xa, xb)
                           : oracle_block_jacobi_step_ex(n, rowptr, col, val, b, R, k, xa, xb, tau, fr);
            } else if (method == ORACLE_GAUSS_SEIDEL) {
                memcpy(xb, xa, sizeof(double) * (size_t)n);
                rc = oracle_gauss_seidel_step(n, rowptr, col, val, b, xb);
            } else {
                rc = -2;
            }
            if (rc != 0) { status = ORACLE_ERR; break; }
            double *t = xa; xa = xb; xb = t;
            rel = oracle_residual_norm(n, rowptr, col, val, b, xa) / bn;
            if (res_hist) res_hist[m] = rel;
            if (!isfinite(rel) || rel > 1e30) { status = ORACLE_DIVERGED; break; }
            if (rel <= tol) break;
        }
        if (m > max_iters) m = max_iters;
    }
    memcpy(x_out, xa, sizeof(double) * (size_t)n);
    *iters_out = m;
    *rel_res_out = rel;
    *converged_out = (status == ORACLE_OK && rel <= tol) ? 1 : 0;
    free(xa); free(xb);
    return status;
}

int oracle_solve(int32_t method, int64_t n, const int32_t *rowptr, const int32_t *col, const double *val,
                 const double *b, const double *x0, double *x_out, int64_t R, int32_t k,
                 int64_t max_iters, double tol, int64_t *iters_out, double *rel_res_out,
                 int32_t *converged_out, double *res_hist) {
    return oracle_solve_ex(method, n, rowptr, col, val, b, x0, x_out, R, k, max_iters, tol, iters_out,
                           rel_res_out, converged_out, res_hist, 1.0, NULL, 0, -1);
}

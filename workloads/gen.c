/*
 * workloads/gen.c — seeded/deterministic INPUT generators shared by the
 * oracle (tests) and the CUDA path (tests, bench).
 *
 * This file holds NONE of the method's arithmetic: it only writes the CSR
 * matrices of the paper's test set (Table 1) or their
 * pattern-exact synthetic stand-ins.
 * Every generator can emit an arbitrary row range [row_lo, row_hi) with GLOBAL
 * column indices, so a multi-GPU rank (or a sampled parity check at full size)
 * can build only the rows it needs.
 *
 * Conventions (all generators):
 *   rowptr  int32[row_hi-row_lo+1], rowptr[0] = 0 (relative to row_lo)
 *   col     int32[nnz_range], strictly ascending within a row, diagonal present
 *   val     double[nnz_range]
 *   return  0 on success, -1 on bad arguments
 *
 * Build: gcc -O2 -fopenmp -fPIC -shared (see __graft_entry__.build()).
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>
#include <math.h>

/* ------------------------------------------------------------------------ */
/* Trefethen_n (Table 1): A = diag(p_1..p_n) + 1 at   */
/* every |i-j| = 2^t < n.  p_i is the i-th prime (p_1 = 2).                   */
/* ------------------------------------------------------------------------ */

/* First `count` primes starting from the `first`-th (0-based) prime. */
static int primes_range(int64_t first, int64_t count, int64_t *out) {
    int64_t need = first + count;
    if (need <= 0) return 0;
    /* upper bound on the need-th prime: n(ln n + ln ln n) for n >= 6 */
    double nd = (double)need;
    int64_t bound = need < 6 ? 15 : (int64_t)(nd * (log(nd) + log(log(nd)))) + 16;
    char *comp = (char *)calloc((size_t)bound + 1, 1);
    if (!comp) return -1;
    int64_t k = 0;
    for (int64_t p = 2; p <= bound && k < need; ++p) {
        if (comp[p]) continue;
        if (k >= first) out[k - first] = p;
        ++k;
        for (int64_t q = p * p; q <= bound; q += p) comp[q] = 1;
    }
    free(comp);
    return k == need ? 0 : -1;
}

static int64_t trefethen_row_nnz(int64_t n, int64_t i) {
    int64_t c = 1;
    for (int64_t o = 1; o < n; o <<= 1) {
        if (i - o >= 0) ++c;
        if (i + o < n) ++c;
    }
    return c;
}

int64_t gen_trefethen_nnz(int64_t n, int64_t row_lo, int64_t row_hi) {
    if (n < 1 || row_lo < 0 || row_hi > n || row_lo > row_hi) return -1;
    int64_t s = 0;
    for (int64_t i = row_lo; i < row_hi; ++i) s += trefethen_row_nnz(n, i);
    return s;
}

int gen_trefethen(int64_t n, int64_t row_lo, int64_t row_hi,
                  int32_t *rowptr, int32_t *col, double *val) {
    if (n < 1 || row_lo < 0 || row_hi > n || row_lo > row_hi) return -1;
    int64_t nr = row_hi - row_lo;
    int64_t *pr = (int64_t *)malloc(sizeof(int64_t) * (size_t)(nr > 0 ? nr : 1));
    if (!pr) return -1;
    if (nr > 0 && primes_range(row_lo, nr, pr) != 0) { free(pr); return -1; }
    int64_t e = 0;
    rowptr[0] = 0;
    for (int64_t r = 0; r < nr; ++r) {
        int64_t i = row_lo + r;
        int64_t offs[64]; int no = 0;
        for (int64_t o = 1; o < n; o <<= 1) offs[no++] = o;
        /* ascending columns: i-2^t for t descending, then i, then i+2^t ascending */
        for (int t = no - 1; t >= 0; --t)
            if (i - offs[t] >= 0) { col[e] = (int32_t)(i - offs[t]); val[e] = 1.0; ++e; }
        col[e] = (int32_t)i; val[e] = (double)pr[r]; ++e;
        for (int t = 0; t < no; ++t)
            if (i + offs[t] < n) { col[e] = (int32_t)(i + offs[t]); val[e] = 1.0; ++e; }
        rowptr[r + 1] = (int32_t)e;
    }
    free(pr);
    return 0;
}

/* ------------------------------------------------------------------------ */
/* 9-point 2D stencil on an m x m grid (fv1/fv2/fv3 pattern, Table 1;  */
/* SURVEY §8(c) P3): row i = x + m*y, off-diagonals `off`, diagonal `diag`.  */
/* ------------------------------------------------------------------------ */

static int64_t s9_row_nnz(int64_t m, int64_t i) {
    int64_t x = i % m, y = i / m;
    int64_t cx = 1 + (x > 0) + (x < m - 1), cy = 1 + (y > 0) + (y < m - 1);
    return cx * cy;
}

int64_t gen_stencil9_2d_nnz(int64_t m, int64_t row_lo, int64_t row_hi) {
    int64_t n = m * m;
    if (m < 1 || row_lo < 0 || row_hi > n || row_lo > row_hi) return -1;
    int64_t s = 0;
    for (int64_t i = row_lo; i < row_hi; ++i) s += s9_row_nnz(m, i);
    return s;
}

int gen_stencil9_2d(int64_t m, double diag, double off, int64_t row_lo, int64_t row_hi,
                    int32_t *rowptr, int32_t *col, double *val) {
    int64_t n = m * m;
    if (m < 1 || row_lo < 0 || row_hi > n || row_lo > row_hi) return -1;
    int64_t nr = row_hi - row_lo;
    int64_t acc = 0;
    rowptr[0] = 0;
    for (int64_t r = 0; r < nr; ++r) { acc += s9_row_nnz(m, row_lo + r); rowptr[r + 1] = (int32_t)acc; }
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < nr; ++r) {
        int64_t i = row_lo + r, x = i % m, y = i / m;
        int64_t e = rowptr[r];
        for (int64_t dy = -1; dy <= 1; ++dy) {
            int64_t yy = y + dy;
            if (yy < 0 || yy >= m) continue;
            for (int64_t dx = -1; dx <= 1; ++dx) {
                int64_t xx = x + dx;
                if (xx < 0 || xx >= m) continue;
                col[e] = (int32_t)(xx + m * yy);
                val[e] = (dx == 0 && dy == 0) ? diag : off;
                ++e;
            }
        }
    }
    return 0;
}

/* ------------------------------------------------------------------------ */
/* 7-point 3D stencil on an m^3 grid (config C5, BASELINE.json configs[4]):   */
/* row i = x + m*y + m*m*z, off-diagonals `off`, diagonal `diag`.            */
/* ------------------------------------------------------------------------ */

static int64_t s7_row_nnz(int64_t m, int64_t i) {
    int64_t x = i % m, y = (i / m) % m, z = i / (m * m);
    return 1 + (x > 0) + (x < m - 1) + (y > 0) + (y < m - 1) + (z > 0) + (z < m - 1);
}

int64_t gen_stencil7_3d_nnz(int64_t m, int64_t row_lo, int64_t row_hi) {
    int64_t n = m * m * m;
    if (m < 1 || row_lo < 0 || row_hi > n || row_lo > row_hi) return -1;
    int64_t s = 0;
#pragma omp parallel for reduction(+ : s) schedule(static)
    for (int64_t i = row_lo; i < row_hi; ++i) s += s7_row_nnz(m, i);
    return s;
}

int gen_stencil7_3d(int64_t m, double diag, double off, int64_t row_lo, int64_t row_hi,
                    int32_t *rowptr, int32_t *col, double *val) {
    int64_t n = m * m * m;
    if (m < 1 || row_lo < 0 || row_hi > n || row_lo > row_hi) return -1;
    int64_t nr = row_hi - row_lo;
    int64_t acc = 0;
    rowptr[0] = 0;
    for (int64_t r = 0; r < nr; ++r) { acc += s7_row_nnz(m, row_lo + r); rowptr[r + 1] = (int32_t)acc; }
    int64_t mm = m * m;
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < nr; ++r) {
        int64_t i = row_lo + r, x = i % m, y = (i / m) % m, z = i / mm;
        int64_t e = rowptr[r];
        /* ascending: -m^2, -m, -1, 0, +1, +m, +m^2 */
        if (z > 0)     { col[e] = (int32_t)(i - mm); val[e] = off; ++e; }
        if (y > 0)     { col[e] = (int32_t)(i - m);  val[e] = off; ++e; }
        if (x > 0)     { col[e] = (int32_t)(i - 1);  val[e] = off; ++e; }
        col[e] = (int32_t)i; val[e] = diag; ++e;
        if (x < m - 1) { col[e] = (int32_t)(i + 1);  val[e] = off; ++e; }
        if (y < m - 1) { col[e] = (int32_t)(i + m);  val[e] = off; ++e; }
        if (z < m - 1) { col[e] = (int32_t)(i + mm); val[e] = off; ++e; }
    }
    return 0;
}

/* Fill helper: out[i] = v (used for b = 1 at the 128M size without numpy temporaries). */
void gen_fill(double *out, int64_t n, double v) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) out[i] = v;
}

/*
 * oracle/mstamp_oracle.c -- TEST INFRASTRUCTURE ONLY.
 *
 * A plain, slow, obviously-correct FP64 CPU implementation of the
 * multi-dimensional matrix profile (mSTAMP) exactly as the paper defines it:
 *
 *   Ju, Raoofy, Yang, Laure, Schulz, "Exploiting Reduced Precision for
 *   GPU-based Time Series Mining", IPDPS 2022.  /root/reference/PAPER.md
 *   cited as PAPER.md:L<n>.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference leg may load this library.  The CUDA product path
 * (paper_conf_ipps_juryl022_b200/) never includes, links or calls it, and
 * this file includes nothing from there.  It deliberately does NOT use the
 * streaming recurrence of Eq. (1): every correlation is a direct dot product
 * of mean-centred windows, so a mistake in the GPU recurrence cannot be
 * mirrored here.
 *
 * Definition implemented (readings G1-G6, G9, G11, G12 of DESIGN.md):
 *   for series s, dimension k, window start i in [0,n), L = n+m-1:
 *     mu[k][i]   = (1/m) sum_t x[k][i+t]                      (two-pass, long double)
 *     norm[k][i] = sqrt( sum_t (x[k][i+t]-mu)^2 )             (population sigma * sqrt(m), G6)
 *   for query window i, reference window j (self-join: skip |i-j| <= excl, G1):
 *     rho_k  = sum_t (xq[k][i+t]-muq)(xr[k][j+t]-mur) / (normq*normr)   (0 if a norm is 0, G4)
 *     rho_k  = clamp(rho_k, -1, 1)                                        (G5)
 *     D_k    = sqrt(2 m (1 - rho_k))                   Eq. (1)
 *     D'     = sort_ascending(D)                       Eq. (2)
 *     D''_k  = (sum_{l<=k} D'_l) / (k+1)               Eq. (2) "inclusive averaging", L523-526 (G11)
 *   P[k][i] = min_j D''_k(i,j),  I[k][i] = smallest j attaining it        Eq. (3), L538-549 (G2, G9)
 *   P2[k][i] = min over j != I[k][i] (the runner-up value; equals P on a tie)
 *   rows with no admissible j: P = +inf, I = -1, P2 = +inf               (G3)
 *
 * Parity pins for every function here live in tests/test_oracle.py.
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---- window statistics (PAPER.md:L509-519 precalculation; two-pass per window) ---- */
int oracle_window_stats(const double* T, int64_t d, int64_t n, int64_t m,
                        double* mu, double* norm)
{
    if (!T || !mu || !norm || d < 1 || n < 1 || m < 2) return 1;
    const int64_t L = n + m - 1;
    for (int64_t k = 0; k < d; ++k) {
        const double* x = T + k * L;
        for (int64_t i = 0; i < n; ++i) {
            long double s = 0.0L;
            for (int64_t t = 0; t < m; ++t) s += (long double)x[i + t];
            long double mean = s / (long double)m;
            long double q = 0.0L;
            for (int64_t t = 0; t < m; ++t) {
                long double c = (long double)x[i + t] - mean;
                q += c * c;
            }
            mu[k * n + i] = (double)mean;
            norm[k * n + i] = (double)sqrtl(q);
        }
    }
    return 0;
}

static int cmp_double(const void* a, const void* b)
{
    double x = *(const double*)a, y = *(const double*)b;
    return (x > y) - (x < y);
}

/* D''_k(i,j) for all k of one cell, from precomputed window stats. */
static void cell_dpp(const double* Tq, const double* Tr, int64_t d, int64_t n, int64_t m,
                     const double* muq, const double* nq, const double* mur, const double* nr,
                     int64_t i, int64_t j, double* Dbuf, double* out)
{
    const int64_t L = n + m - 1;
    for (int64_t k = 0; k < d; ++k) {
        const double* xq = Tq + k * L + i;
        const double* xr = Tr + k * L + j;
        const double mq = muq[k * n + i], mr = mur[k * n + j];
        double qt = 0.0;
        for (int64_t t = 0; t < m; ++t) qt += (xq[t] - mq) * (xr[t] - mr);
        const double den = nq[k * n + i] * nr[k * n + j];
        double rho = (den > 0.0) ? qt / den : 0.0;
        if (rho > 1.0) rho = 1.0;
        if (rho < -1.0) rho = -1.0;
        Dbuf[k] = sqrt(2.0 * (double)m * (1.0 - rho));
    }
    qsort(Dbuf, (size_t)d, sizeof(double), cmp_double);
    double s = 0.0;
    for (int64_t k = 0; k < d; ++k) {
        s += Dbuf[k];
        out[k] = s / (double)(k + 1);
    }
}

/* One cell, all k: out[k] = D''_k(i,j).  Tr == NULL means self-join (Tr = Tq). */
int oracle_cell(const double* Tq, const double* Tr, int64_t d, int64_t n, int64_t m,
                int64_t i, int64_t j, double* out)
{
    if (!Tq || !out || d < 1 || n < 1 || m < 2 || i < 0 || i >= n || j < 0 || j >= n) return 1;
    if (!Tr) Tr = Tq;
    double* muq = malloc(sizeof(double) * d * n);
    double* nq = malloc(sizeof(double) * d * n);
    double* mur = malloc(sizeof(double) * d * n);
    double* nr = malloc(sizeof(double) * d * n);
    double* Db = malloc(sizeof(double) * d);
    if (!muq || !nq || !mur || !nr || !Db) { free(muq); free(nq); free(mur); free(nr); free(Db); return 2; }
    oracle_window_stats(Tq, d, n, m, muq, nq);
    oracle_window_stats(Tr, d, n, m, mur, nr);
    cell_dpp(Tq, Tr, d, n, m, muq, nq, mur, nr, i, j, Db, out);
    free(muq); free(nq); free(mur); free(nr); free(Db);
    return 0;
}

/* Many cells: out[c*d + k] = D''_k(ii[c], jj[c]); stats computed once. */
int oracle_cells(const double* Tq, const double* Tr, int64_t d, int64_t n, int64_t m,
                 const int64_t* ii, const int64_t* jj, int64_t count, double* out)
{
    if (!Tq || !ii || !jj || !out || d < 1 || n < 1 || m < 2 || count < 0) return 1;
    for (int64_t c = 0; c < count; ++c)
        if (ii[c] < 0 || ii[c] >= n || jj[c] < 0 || jj[c] >= n) return 1;
    if (!Tr) Tr = Tq;
    double* muq = malloc(sizeof(double) * d * n);
    double* nq = malloc(sizeof(double) * d * n);
    double* mur = malloc(sizeof(double) * d * n);
    double* nr = malloc(sizeof(double) * d * n);
    double* Db = malloc(sizeof(double) * d);
    if (!muq || !nq || !mur || !nr || !Db) { free(muq); free(nq); free(mur); free(nr); free(Db); return 2; }
    oracle_window_stats(Tq, d, n, m, muq, nq);
    oracle_window_stats(Tr, d, n, m, mur, nr);
    for (int64_t c = 0; c < count; ++c)
        cell_dpp(Tq, Tr, d, n, m, muq, nq, mur, nr, ii[c], jj[c], Db, out + c * d);
    free(muq); free(nq); free(mur); free(nr); free(Db);
    return 0;
}

typedef struct {
    const double *Tq, *Tr, *muq, *nq, *mur, *nr;
    int64_t d, n, m, excl, self;
    const int64_t* rows;
    int64_t nrows;
    int64_t r_begin, r_end;
    double *P, *P2;
    int64_t* I;
} job_t;

static void* worker(void* arg)
{
    job_t* jb = (job_t*)arg;
    const int64_t d = jb->d, n = jb->n, nrows = jb->nrows;
    double* Db = malloc(sizeof(double) * d);
    double* v = malloc(sizeof(double) * d);
    double* best = malloc(sizeof(double) * d);
    double* best2 = malloc(sizeof(double) * d);
    int64_t* idx = malloc(sizeof(int64_t) * d);
    for (int64_t r = jb->r_begin; r < jb->r_end; ++r) {
        const int64_t i = jb->rows ? jb->rows[r] : r;
        for (int64_t k = 0; k < d; ++k) { best[k] = INFINITY; best2[k] = INFINITY; idx[k] = -1; }
        for (int64_t j = 0; j < n; ++j) {
            if (jb->self && llabs(i - j) <= jb->excl) continue; /* exclusion zone, G1 */
            cell_dpp(jb->Tq, jb->Tr, d, n, jb->m, jb->muq, jb->nq, jb->mur, jb->nr, i, j, Db, v);
            for (int64_t k = 0; k < d; ++k) {      /* Eq. (3): strict <, ascending j => lowest j wins ties */
                if (v[k] < best[k]) { best2[k] = best[k]; best[k] = v[k]; idx[k] = j; }
                else if (v[k] < best2[k]) { best2[k] = v[k]; }
            }
        }
        for (int64_t k = 0; k < d; ++k) {
            jb->P[k * nrows + r] = best[k];
            jb->P2[k * nrows + r] = best2[k];
            jb->I[k * nrows + r] = idx[k];
        }
    }
    free(Db); free(v); free(best); free(best2); free(idx);
    return NULL;
}

/*
 * Full (rows == NULL, nrows == n) or sampled (rows[0..nrows)) matrix profile.
 * T: d x L row-major (dimension k contiguous).  Tr == NULL -> self-join with
 * exclusion zone |i-j| <= excl; otherwise AB-join (excl ignored).
 * Outputs are d x nrows: P[k*nrows + r], P2[...], I[...] for query rows[r].
 */
int oracle_mstamp(const double* Tq, const double* Tr, int64_t d, int64_t n, int64_t m,
                  int64_t excl, const int64_t* rows, int64_t nrows, int nthreads,
                  double* P, int64_t* I, double* P2)
{
    if (!Tq || !P || !I || !P2 || d < 1 || n < 1 || m < 2 || nrows < 0) return 1;
    if (!rows && nrows != n) return 1;
    const int self = (Tr == NULL);
    if (self) Tr = Tq;
    if (nthreads < 1) nthreads = 1;
    double* muq = malloc(sizeof(double) * d * n);
    double* nq = malloc(sizeof(double) * d * n);
    double* mur = self ? muq : malloc(sizeof(double) * d * n);
    double* nr = self ? nq : malloc(sizeof(double) * d * n);
    if (!muq || !nq || !mur || !nr) return 2;
    oracle_window_stats(Tq, d, n, m, muq, nq);
    if (!self) oracle_window_stats(Tr, d, n, m, mur, nr);

    pthread_t* th = malloc(sizeof(pthread_t) * nthreads);
    job_t* jobs = malloc(sizeof(job_t) * nthreads);
    for (int t = 0; t < nthreads; ++t) {
        jobs[t] = (job_t){Tq, Tr, muq, nq, mur, nr, d, n, m, excl, self, rows, nrows,
                          nrows * t / nthreads, nrows * (t + 1) / nthreads, P, P2, I};
        pthread_create(&th[t], NULL, worker, &jobs[t]);
    }
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    free(th); free(jobs);
    free(muq); free(nq);
    if (!self) { free(mur); free(nr); }
    return 0;
}

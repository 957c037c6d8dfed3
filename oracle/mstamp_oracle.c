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
 *   oracle_mstamp_band: the same min over the cells of one diagonal band only (the
 *   per-GPU partial of SURVEY 8(e)), for sampled rows of full-size configs.
 *
 * Parity pins for every function here live in tests/test_oracle.py.
 */
#include <math.h>
#include <pthread.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ---- window statistics (PAPER.md:L509-519 precalculation; two-pass per window) ---- */
static void window_stat(const double* x, int64_t m, double* mu, double* norm)
{
    long double s = 0.0L;
    for (int64_t t = 0; t < m; ++t) s += (long double)x[t];
    long double mean = s / (long double)m;
    long double q = 0.0L;
    for (int64_t t = 0; t < m; ++t) {
        long double c = (long double)x[t] - mean;
        q += c * c;
    }
    *mu = (double)mean;
    *norm = (double)sqrtl(q);
}

int oracle_window_stats(const double* T, int64_t d, int64_t n, int64_t m,
                        double* mu, double* norm)
{
    if (!T || !mu || !norm || d < 1 || n < 1 || m < 2) return 1;
    const int64_t L = n + m - 1;
    for (int64_t k = 0; k < d; ++k)
        for (int64_t i = 0; i < n; ++i)
            window_stat(T + k * L + i, m, &mu[k * n + i], &norm[k * n + i]);
    return 0;
}

static int cmp_double(const void* a, const void* b)
{
    double x = *(const double*)a, y = *(const double*)b;
    return (x > y) - (x < y);
}

/* D''_k(i,j) for all k of one cell; mq/nq/mr/nr hold the d window stats of windows i
 * (query) and j (reference) (stride sq / sr between dimensions). */
static void dpp_core(const double* Tq, const double* Tr, int64_t d, int64_t n, int64_t m,
                     const double* mq_, int64_t sq, const double* nq_, const double* mr_, int64_t sr,
                     const double* nr_, int64_t i, int64_t j, double* Dbuf, double* out)
{
    const int64_t L = n + m - 1;
    for (int64_t k = 0; k < d; ++k) {
        const double* xq = Tq + k * L + i;
        const double* xr = Tr + k * L + j;
        const double mq = mq_[k * sq], mr = mr_[k * sr];
        double qt = 0.0;
        for (int64_t t = 0; t < m; ++t) qt += (xq[t] - mq) * (xr[t] - mr);
        const double den = nq_[k * sq] * nr_[k * sr];
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

/* D''_k(i,j) for all k of one cell, from precomputed (d x n) window stats. */
static void cell_dpp(const double* Tq, const double* Tr, int64_t d, int64_t n, int64_t m,
                     const double* muq, const double* nq, const double* mur, const double* nr,
                     int64_t i, int64_t j, double* Dbuf, double* out)
{
    dpp_core(Tq, Tr, d, n, m, muq + i, n, nq + i, mur + j, n, nr + j, i, j, Dbuf, out);
}

/* The d window stats of window i of T (two-pass per window, as oracle_window_stats). */
static void stats_of(const double* T, int64_t d, int64_t n, int64_t m, int64_t i, double* mu, double* nrm)
{
    const int64_t L = n + m - 1;
    for (int64_t k = 0; k < d; ++k) window_stat(T + k * L + i, m, &mu[k], &nrm[k]);
}

/* One cell, all k: out[k] = D''_k(i,j).  Tr == NULL means self-join (Tr = Tq). */
int oracle_cells(const double* Tq, const double* Tr, int64_t d, int64_t n, int64_t m,
                 const int64_t* ii, const int64_t* jj, int64_t count, double* out);
int oracle_cell(const double* Tq, const double* Tr, int64_t d, int64_t n, int64_t m,
                int64_t i, int64_t j, double* out)
{
    if (!Tq || !out || d < 1 || n < 1 || m < 2 || i < 0 || i >= n || j < 0 || j >= n) return 1;
    return oracle_cells(Tq, Tr, d, n, m, &i, &j, 1, out);
}

/* Many cells: out[c*d + k] = D''_k(ii[c], jj[c]); the stats of each cell's two windows are
 * computed where needed (identical arithmetic to oracle_window_stats). */
int oracle_cells(const double* Tq, const double* Tr, int64_t d, int64_t n, int64_t m,
                 const int64_t* ii, const int64_t* jj, int64_t count, double* out)
{
    if (!Tq || !ii || !jj || !out || d < 1 || n < 1 || m < 2 || count < 0) return 1;
    for (int64_t c = 0; c < count; ++c)
        if (ii[c] < 0 || ii[c] >= n || jj[c] < 0 || jj[c] >= n) return 1;
    if (!Tr) Tr = Tq;
    double* st = malloc(sizeof(double) * 5 * d);
    if (!st) return 2;
    double *mq = st, *nq = st + d, *mr = st + 2 * d, *nr = st + 3 * d, *Db = st + 4 * d;
    for (int64_t c = 0; c < count; ++c) {
        stats_of(Tq, d, n, m, ii[c], mq, nq);
        stats_of(Tr, d, n, m, jj[c], mr, nr);
        dpp_core(Tq, Tr, d, n, m, mq, 1, nq, mr, 1, nr, ii[c], jj[c], Db, out + c * d);
    }
    free(st);
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

/*
 * Partial profile of one diagonal band (the unit a GPU rank computes before the
 * MINLOC merge): for query rows[r], the min / argmin / runner-up over the cells (i, j) of the
 * band's diagonals delta in [dlo, dhi):  AB-join j - i = delta;  self-join |j - i| = delta
 * (each unordered pair once per band, applied to row and column, reading G13), still
 * skipping |i - j| <= excl (G1).  Same per-cell arithmetic and the same ascending-j strict-<
 * rule as oracle_mstamp; window stats computed per window where needed, so full-size configs
 * (n = 2^21) cost O(#rows * band width * d * m), not O(n * d * m).
 */
typedef struct {
    const double *Tq, *Tr;
    int64_t d, n, m, excl, self, dlo, dhi;
    const int64_t* rows;
    int64_t nrows, r_begin, r_end;
    double *P, *P2;
    int64_t* I;
} band_job_t;

static void* band_worker(void* arg)
{
    band_job_t* jb = (band_job_t*)arg;
    const int64_t d = jb->d, n = jb->n, nrows = jb->nrows;
    double* buf = malloc(sizeof(double) * 9 * d);
    int64_t* idx = malloc(sizeof(int64_t) * d);
    double *mq = buf, *nq = buf + d, *mr = buf + 2 * d, *nr = buf + 3 * d, *Db = buf + 4 * d;
    double *v = buf + 5 * d, *best = buf + 6 * d, *best2 = buf + 7 * d;
    for (int64_t r = jb->r_begin; r < jb->r_end; ++r) {
        const int64_t i = jb->rows[r];
        for (int64_t k = 0; k < d; ++k) { best[k] = INFINITY; best2[k] = INFINITY; idx[k] = -1; }
        stats_of(jb->Tq, d, n, jb->m, i, mq, nq);
        for (int64_t j = 0; j < n; ++j) {
            const int64_t delta = jb->self ? llabs(j - i) : j - i;
            if (delta < jb->dlo || delta >= jb->dhi) continue;
            if (jb->self && llabs(i - j) <= jb->excl) continue; /* exclusion zone, G1 */
            stats_of(jb->Tr, d, n, jb->m, j, mr, nr);
            dpp_core(jb->Tq, jb->Tr, d, n, jb->m, mq, 1, nq, mr, 1, nr, i, j, Db, v);
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
    free(buf); free(idx);
    return NULL;
}

int oracle_mstamp_band(const double* Tq, const double* Tr, int64_t d, int64_t n, int64_t m,
                       int64_t excl, const int64_t* rows, int64_t nrows, int64_t dlo, int64_t dhi,
                       int nthreads, double* P, int64_t* I, double* P2)
{
    if (!Tq || !rows || !P || !I || !P2 || d < 1 || n < 1 || m < 2 || nrows < 0) return 1;
    for (int64_t r = 0; r < nrows; ++r)
        if (rows[r] < 0 || rows[r] >= n) return 1;
    const int self = (Tr == NULL);
    if (self) Tr = Tq;
    if (nthreads < 1) nthreads = 1;
    if (nthreads > nrows && nrows > 0) nthreads = (int)nrows;
    pthread_t* th = malloc(sizeof(pthread_t) * nthreads);
    band_job_t* jobs = malloc(sizeof(band_job_t) * nthreads);
    for (int t = 0; t < nthreads; ++t) {
        jobs[t] = (band_job_t){Tq, Tr, d, n, m, excl, self, dlo, dhi, rows, nrows,
                               nrows * t / nthreads, nrows * (t + 1) / nthreads, P, P2, I};
        pthread_create(&th[t], NULL, band_worker, &jobs[t]);
    }
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    free(th); free(jobs);
    return 0;
}

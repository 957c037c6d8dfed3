// Internal interface between the host scheduler (mp_api.cpp) and the CUDA kernels
// (mp_kernels.cu).  Not part of the C ABI.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace mpk {

// Parameters of the fused diagonal kernel (one launch = a contiguous tile range).
struct MainParams {
    const void* st_q;   // stats, position-major [pos][dim], V4 = (df, dg, a, 0)   (query / rows)
    const void* st_r;   // stats of the reference series (columns); == st_q for self-join
    const void* tw_q;   // working-precision series, position-major padded [t][Dp], t < L (seeds)
    const void* tw_r;
    const void* mu_q;   // working-precision window means, position-major padded [pos][Dp]
    const void* mu_r;
    void* keys;         // merge keys [pos][rank] of the QUERY profile (self-join: the one profile)
    // tile order.  order == 1, segment-major (warp-tile kernels): all of the band's diagonal
    // blocks of row segment q, then q + 1, ...; tile t (0 <= t < t_count) is block
    // q_block0[q] + (t - q_prefix[q]) of segment q, q_prefix[q] <= t < q_prefix[q + 1].
    // order == 0, block-major (block-cooperative kernels): tile t_begin + t lies in block b
    // with seg_prefix[b] <= t_begin + t < seg_prefix[b + 1], segment rlo_b / HT + (that - seg_prefix[b]).
    int order;
    const long long* q_prefix;    // exclusive prefix of #tiles per row segment (nq + 1)
    const long long* q_block0;    // first diagonal block of the band in segment q (nq)
    long long nq;                 // number of row segments (ceil(n / HT))
    const long long* seg_prefix;  // exclusive prefix of #segments per diagonal block (nb + 1)
    long long nb, t_begin;
    long long t_count;            // tiles of this launch (the rank's band)
    unsigned long long* counter;  // zeroed before launch
    long long n;                  // subsequences
    int d, m, H;                  // dims, window, re-seed interval H (rows)
    int HT;                       // tile height (multiple of H)
    long long delta_lo, delta_hi; // diagonal range [lo, hi] (j = i + delta)
    long long q_lo;               // block-major order: first row segment of the launch's row
                                  // window (0; > 0 only for a streamed chunk, mp_compute_stream)
    // tensor-core seed table (half block kernels, mp_config.seed_mode = MP_SEEDS_TC): seeds of
    // rows r H, r in [tab_r_lo, tab_r_hi), columns [tab_j_lo, tab_j_lo + tab_ldj) at
    // seed_tab[((r - tab_r_lo) * d + dim) * tab_ldj + (j - tab_j_lo)]; nullptr: direct seeds
    const void* seed_tab;
    long long tab_r_lo, tab_r_hi, tab_j_lo, tab_ldj;
};

// Tensor-core seed GEMM (mp_seed_tc.cu): seeds of rows r H, r in [r_lo, r_hi), against columns
// [j_lo, j_hi) for every dimension, from the FP64 input scaled by the per-dimension power of two
// (reading G16) and the FP32 window means of the Mixed precalc.
struct SeedParams {
    const double* Tq;      // query series [dim][L]
    const double* Tr;      // reference series (== Tq for a self-join)
    const double* scale_q; // [d]
    const double* scale_r;
    const float* mu_q;     // window means [dim][n] (FP32)
    const float* mu_r;
    void* tab;             // out (half): [(r - r_lo) * d + dim][ldj]
    long long n;
    int d, m, H;
    long long r_lo, r_hi, j_lo, j_hi, ldj;   // ldj: a multiple of 8, >= j_hi - j_lo
};

struct PreParams {
    const double* T;    // input [dim][t] FP64, L = n + m - 1
    void* st;           // out stats [pos][dim]
    void* tw;           // out working series, position-major padded [t][Dp], t < L (seeds)
    void* mu;           // out window mean [dim][pos]
    void* mup;          // out window mean, position-major padded [pos][Dp] (seeds)
    int Dp;             // padded dimension count of the kernel variant (DL * G)
    int pm_G, pm_DL;    // pm_G > 0: the seed operands (tw, mup) store dim kk*G + g at g*DL + kk, so
                        // each lane's DL dims are contiguous (mp_diag_ctab); 0: natural order
    float* nrm32;       // scratch for FP32 path (norm) [dim][pos]
    double* nrm64;
    long long n;
    int d, m;
    // position window (mp_compute_stream; a full run: w0 = 0, w1 = n, T_off = s_off = 0,
    // T_ld = L, s_ld = n).  Outputs at absolute positions (st, st_pair, tw, mup) are written for
    // positions [w0, w1) (tw: t in [w0, w1 + m - 1); st_pair: entries [w0, w1]).  T holds
    // x[dim][t] at T[dim * T_ld + t - T_off]; the per-window scratch (mu, nrm, flat) holds
    // position pos at (pos - s_off) with leading dimension s_ld and covers [s_off, s_end).
    long long w0, w1, T_off, T_ld, s_off, s_end, s_ld;
    // FP16 / Mixed only
    void* st_pair;      // out stats in pair format [pos][dim] (x_pos, x_pos+1) half2 x 4
    double* scale;      // scratch [d]: exact power-of-two per-dimension scale (reading G16)
    unsigned long long* maxbits;  // scratch [2 d]: max window norm, max |x| (double bits)
    void* flat;         // scratch [3][pos][dim] half: df, dg, a
};

// Precision codes match mp_precision.
// P32N (kernel-internal): FP32 with the plain QT recurrence, chosen for short windows (warp kernels)
enum { P64 = 0, P32 = 1, P16 = 2, PMIX = 3, P16C = 4, P16CK = 5, P32N = 6 };

// Variant selection for a given (precision, d): dims per lane DL and lanes per cell G.
struct Variant { int DL; int G; int W; int NC; int cta = 0; /* warps per block of the block-cooperative kernel, 0: warp tiles */
                 bool ctab = false; /* FP32 block-cooperative kernel with TMA staging (mp_diag_ctab) */ };
Variant pick_variant(int prec, int d);
size_t smem_per_block(int prec, int d, bool self);
int variant_warps_per_block(int prec, int d, bool self);

// Launchers (return cudaError_t).
cudaError_t launch_precompute(int prec, const PreParams& p, cudaStream_t s, bool with_scale = true);
// half modes: per-dimension scale (reading G16) over a window [w0, w1) (reset: clear the maxima
// first), then pick the scales; mp_compute_stream runs these over every window before the chunks
cudaError_t launch_scale_max(const PreParams& p, bool reset, cudaStream_t s);
cudaError_t launch_scale_pick(int prec, const PreParams& p, cudaStream_t s);
// streamed finalize: keys (internal format, absolute positions) of positions [p0, p1) -> P, I
// window buffers [rank][p1 - p0]
cudaError_t launch_finalize_window(int prec, const void* keys, long long p0, long long p1, int d, double* P,
                                   long long* I, cudaStream_t s);
cudaError_t launch_init_keys(int prec, void* keys, long long count, cudaStream_t s);
cudaError_t launch_main(int prec, bool self, const MainParams& p, int grid, cudaStream_t s);
int main_blocks_per_sm(int prec, int d, bool self);
cudaError_t launch_finalize(int prec, const void* keys_ext, long long n, int d, double* P,
                            long long* I, cudaStream_t s);
cudaError_t launch_keys_to_ext(int prec, const void* keys, void* ext, long long count,
                               cudaStream_t s);
cudaError_t launch_key_mask(long long count, long long* ext, const long long* gv, cudaStream_t s);
cudaError_t launch_check_finite(const double* x, long long count, int* flag, cudaStream_t s);
cudaError_t launch_seed_gemm(const SeedParams& p, cudaStream_t s);
// stage self-tests (include/mp.h)
cudaError_t launch_selftest_sort_scan(int d, long long count, const float* in, float* out, cudaStream_t s);
cudaError_t launch_selftest_unpack(int prec, const void* st, long long n, int d, double* df, double* dg, double* a,
                                   cudaStream_t s);

}  // namespace mpk

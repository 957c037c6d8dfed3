/*
 * include/mp.h -- C ABI of the B200-native mSTAMP hot path (libmstamp_b200.so).
 *
 * What it computes (PAPER.md = /root/reference/PAPER.md, Ju et al., IPDPS 2022):
 *   For query series Tq and reference series Tr (both d x L, L = n + m - 1,
 *   PAPER.md:L461-473, footnote L515-516: n = number of subsequences), for every
 *   cell (i, j) of the n x n subsequence grid and every dimension k:
 *     QT  by the streaming recurrence along each diagonal        Eq. (1)
 *     D   = sqrt(2 m (1 - QT d_q^-1 d_r^-1))                     Eq. (1)
 *     D'  = sort(D[i,j,:]) ascending;  D'' = inclusive mean      Eq. (2)
 *     P[k][i] = min_j D''[i,j,k],  I[k][i] = argmin_j            Eq. (3)
 *   Self-join (Tr == NULL): cells with |i - j| <= exclusion are skipped
 *   (reading G1); AB-join: every j, query profile only.
 *   Ties: the lowest j wins (G2).  Rows with no admissible j: P = +inf, I = -1 (G3).
 *
 * Layouts: every matrix is row-major "d rows x n (or L) columns", i.e. element
 *   (k, i) at [k * n + i]; dimension k contiguous (the paper's "dimension-wise
 *   layout", L662-666).
 * Precision modes (Fig. 1 table, Sec. III-C): see mp_precision.
 * Ownership: the caller owns T, Tr, P, I (host memory for mp_compute, device memory
 *   for the _device variants); the context owns all device scratch and the
 *   per-device streams it creates, caches scratch by shape, frees it in mp_free.
 * Errors: every call returns mp_status; nothing aborts or throws across the ABI.
 *   On a non-OK status outputs are unspecified and no memory is leaked;
 *   mp_last_error(ctx) returns a message.
 * Threading: one context per host thread.
 * Determinism: for a given (inputs, prec, reseed interval) the outputs are
 *   bit-identical for any number of GPUs / ranks and any launch order (fixed
 *   tiling; lexicographic (value, index) minimum is order-independent).
 */
#ifndef MP_H_
#define MP_H_

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
    MP_OK = 0,
    MP_ERR_INVALID = 1,     /* bad argument: NULL, d<1, n<2, m<2, non-finite input, n >= 2^31, d > MP_MAX_D */
    MP_ERR_NOMEM = 2,       /* device or host allocation failed */
    MP_ERR_CUDA = 3,        /* CUDA runtime error (message in mp_last_error) */
    MP_ERR_NCCL = 4,        /* reserved: collectives run in the caller's process group */
    MP_ERR_UNSUPPORTED = 5  /* valid request this build does not implement (e.g. precision x d) */
} mp_status;

typedef enum {
    MP_FP64 = 0,   /* precalculation FP64, main loop FP64           (L426-428, L764-766) */
    MP_FP32 = 1,   /* precalculation FP32, main loop FP32           (L430-432, L771-772) */
    MP_FP16 = 2,   /* precalculation FP16, main loop FP16           (L434-436, L773-776) */
    MP_MIXED = 3,  /* precalculation FP32 (plain sums), main loop FP16 (L438-440, L777-785) */
    MP_FP16C = 4,  /* precalculation FP16 with Kahan-compensated sums, main loop FP16
                      (Fig. 1 "FP16 with compensator" L442-444; G17, Fig. 1 reading) */
    MP_FP16CK = 5  /* FP16C, the text's reading: precalculation (window statistics and seeds) in
                      FP32 arithmetic with Kahan-compensated sums, main loop FP16 (L786-798
                      "higher precision mode in precalculation ... Kahan's compensated
                      summation"; G17, text reading).  Re-seed interval of MIXED. */
} mp_precision;

#define MP_MAX_D 1024

typedef struct mp_ctx mp_ctx;   /* opaque */

typedef struct {
    int device;             /* CUDA device ordinal this context drives (one process per GPU) */
    int64_t reseed_h[4];    /* re-seed interval H (rows) for FP64, FP32, FP16 (also FP16C), MIXED
                               (also FP16CK);
                               0 -> default (R2); rounded up to a multiple of 8 (re-seeds
                               fall on staging-batch starts); < 0 or > 2^30 -> MP_ERR_INVALID */
    int seed_mode;          /* how the QT seeds of MIXED / FP16CK are computed:
                               MP_SEEDS_DIRECT (0): per-cell dot products on the CUDA cores, in
                               FP32; MP_SEEDS_TC (1): one tensor-core GEMM per row chunk
                               (tcgen05, FP16 operands, FP32 accumulation; SURVEY 8(f) NEXT-3,
                               PAPER.md:L2433-2434) for the block kernels (d >= 64), written to a
                               seed table the fused kernel reads.  Other precisions ignore it.
                               Other values -> MP_ERR_INVALID. */
} mp_config;

#define MP_SEEDS_DIRECT 0
#define MP_SEEDS_TC 1

/* Create a context on cfg->device (cfg == NULL -> device 0, defaults). */
mp_status mp_init(mp_ctx** out, const mp_config* cfg);

/* Free all device memory and streams owned by ctx.  NULL-safe. */
void mp_free(mp_ctx* ctx);

/* Message for the last non-OK status on ctx (static string if ctx == NULL). */
const char* mp_last_error(const mp_ctx* ctx);

/* Library version string. */
const char* mp_version(void);

/*
 * Whole matrix profile on the context's device, HOST buffers.
 *   T   [d x L] query series (FP64, L = n + m - 1); Tr: reference series, same
 *       shape, or NULL for a self-join.
 *   exclusion: self-join skips |i - j| <= exclusion; < 0 -> ceil(m / 4); ignored for AB.
 *   P   [d x n] out: P[k*n + i] = mean of the k+1 smallest per-dimension distances
 *       of query window i to its nearest reference window.
 *   I   [d x n] out: that reference window's index j, or -1 if none.
 * Includes the host->device copy of T (and Tr) and the device->host copy of P, I.
 */
mp_status mp_compute(mp_ctx* ctx, const double* T, const double* Tr,
                     int64_t d, int64_t n, int64_t m, mp_precision prec,
                     int64_t exclusion, double* P, int64_t* I);

/* Same as mp_compute with DEVICE pointers, enqueued on the caller's CUDA stream (NULL = the
 * legacy default stream).  Returns after enqueueing (one host sync for the input check). */
mp_status mp_compute_device(mp_ctx* ctx, void* cuda_stream, const double* dT, const double* dTr,
                            int64_t d, int64_t n, int64_t m, mp_precision prec,
                            int64_t exclusion, double* dP, int64_t* dI);

/*
 * Multi-GPU building blocks (one process per GPU; the caller's process group does
 * the collective -- the only exchange step of the path, Pseudocode 2 l.6-8,
 * PAPER.md:L738-740, replaced by an on-device MINLOC all-reduce).
 *
 * mp_partial_device: compute the band `rank` of `world` equal-cell diagonal
 *   bands and leave the partial profile as merge keys in dKeys.
 *   dKeys must hold mp_key_words(d, n, prec) int64 words on the device.
 *   Key format (bit-exact lexicographic (value, index) order):
 *     FP32/FP16/MIXED: one int64 per (k, i) = (float bits of the k-dim distance SUM << 32) | j;
 *                      reduce with MIN over int64.
 *     FP64: two int64 planes; plane 0 = double bits of the distance SUM (reduce MIN),
 *           plane 1 = index; call mp_key_mask_device between the two MIN reductions.
 *   Empty entries: FP32 keys >= 0x7F80000000000000 (value +inf); FP64 index plane INT64_MAX.
 */
int64_t   mp_key_words(int64_t d, int64_t n, mp_precision prec);
mp_status mp_partial_device(mp_ctx* ctx, void* cuda_stream, const double* dT, const double* dTr,
                            int64_t d, int64_t n, int64_t m, mp_precision prec, int64_t exclusion,
                            int rank, int world, int64_t* dKeys);
/* FP64 merge step 2: where plane0 != global plane0 (dGlobalV), set the index to INT64_MAX. */
mp_status mp_key_mask_device(mp_ctx* ctx, void* cuda_stream, int64_t d, int64_t n,
                             int64_t* dKeys, const int64_t* dGlobalV);
/* Merged keys -> P (double, divided by k+1) and I (int64, -1 for empty). */
mp_status mp_finalize_device(mp_ctx* ctx, void* cuda_stream, int64_t d, int64_t n, mp_precision prec,
                             const int64_t* dKeys, double* dP, int64_t* dI);

/*
 * Host-side scheduler query (no GPU needed): the first diagonal-block index of
 * band `rank` of `world` and the number of cells per band (cells = (i,j) pairs
 * the band computes).  Bands are contiguous diagonal ranges with equal cell
 * counts up to one block.  block_begin/cells arrays have world+1 / world entries.
 */
mp_status mp_plan_bands(int64_t d, int64_t n, int64_t m, mp_precision prec, int64_t exclusion,
                        int self_join, int world, int64_t* block_begin, int64_t* cells);

/* Diagonal range of each band: band g covers diagonals delta = j - i in
 * [diag_begin[g], diag_begin[g+1]) (world+1 entries; self-join delta > exclusion, AB-join
 * delta in (-n, n)).  Host only, no GPU needed. */
mp_status mp_plan_diagonals(int64_t d, int64_t n, int64_t m, mp_precision prec, int64_t exclusion,
                            int self_join, int world, int64_t* diag_begin);

/* Kernel timing of the last mp_compute* / mp_partial_device call on ctx (ms, CUDA
 * events around the main diagonal kernel only) and its launch count. */
mp_status mp_last_timing(const mp_ctx* ctx, double* main_kernel_ms, int64_t* launches);

/*
 * Beyond-memory streaming (the tiling "decouples the size
 * of the distance matrix" from "the limited device memory", and L2432-2433).
 *
 * mp_compute_stream: the same result as mp_compute -- bit-identical P and I for every precision
 *   -- computed with at most about `device_bytes` of device memory for the per-position arrays
 *   (statistics, seed operands, merge keys), independent of n.  T, Tr, P, I and the running merge
 *   keys stay in host memory (the library allocates a pinned key store of n*d*8 bytes, n*d*16
 *   for FP64, for the duration of the call).  The tile plan is cut into row chunks of R rows
 *   (a multiple of the tile height) times diagonal bands of Wb diagonals; per step the device
 *   holds one row window and one column window (CUDA virtual memory: full-size address
 *   reservations, physical memory mapped for the windows only), computes the window statistics
 *   from a T slice, restores / saves the keys of the windows, and finalizes rows [i0, i1) when
 *   their chunk is done.  Arguments as mp_compute; device_bytes > 0.  Errors: MP_ERR_NOMEM when
 *   device_bytes cannot hold one row segment of the plan; MP_ERR_UNSUPPORTED when the driver
 *   lacks the virtual-memory entry points.  Scratch cached on ctx by other calls is not counted.
 *   Testing knobs: the environment variables MP_STREAM_ROWS / MP_STREAM_DIAGS override R / Wb
 *   (rounded up to the tile height / block width) so small inputs exercise many chunks.
 * mp_plan_stream: the chunk geometry (rows per chunk R, diagonals per band Wb) mp_compute_stream
 *   chooses for a budget and an allocation granularity (bytes; the device's is 2 MiB).  Host
 *   only, no GPU needed.  MP_ERR_NOMEM as above.
 * mp_last_stream_info: R, Wb, the peak physically mapped bytes and the number of fused-kernel
 *   launches of the last mp_compute_stream on ctx (mp_last_timing gives the summed kernel time).
 */
mp_status mp_compute_stream(mp_ctx* ctx, const double* T, const double* Tr, int64_t d, int64_t n, int64_t m,
                            mp_precision prec, int64_t exclusion, int64_t device_bytes, double* P, int64_t* I);
mp_status mp_plan_stream(int64_t d, int64_t n, int64_t m, mp_precision prec, int64_t exclusion, int self_join,
                         int64_t device_bytes, int64_t granularity, int64_t* rows_per_chunk,
                         int64_t* diagonals_per_band);
mp_status mp_last_stream_info(const mp_ctx* ctx, int64_t* rows_per_chunk, int64_t* diagonals_per_band,
                              int64_t* peak_device_bytes, int64_t* launches);

/*
 * Stage self-tests (per-stage unit tests of SURVEY 4; tests/test_gpu_stages.py).  They run ONE
 * stage of the hot path on the device with the same device code the fused kernels use, on host
 * buffers (copies in and out included), so a stage can be checked against the oracle / numpy in
 * isolation.  Not part of the compute path.
 *
 * mp_selftest_sort_scan: for each of `count` cells, the FP32 kernel variant chosen for `d`
 *   (warp tiles for d <= 32, block-cooperative tiles above: the same sort network, cross-lane
 *   merge and fused scan templates) sorts the cell's d values ascending and writes the inclusive
 *   prefix sums S_k = sum of the k+1 smallest (Eq. 2).  in / out: count x d
 *   floats, cell-major.  Values may be any non-negative float, +inf or denormal.
 * mp_selftest_precompute: the precalculation of mode `prec` (readings G7,
 *   R1') on T (d x L, L = n + m - 1): writes df, dg, a (each n x d, position-major, as doubles;
 *   half modes: the unscaled values divided back by the per-dimension power-of-two scale are NOT
 *   returned -- FP64 and FP32 only).
 */
mp_status mp_selftest_sort_scan(mp_ctx* ctx, int64_t d, int64_t count, const float* in, float* out);
/* mp_selftest_seeds: the tensor-core seed GEMM (MP_SEEDS_TC) alone: after the MIXED / FP16CK
 *   precalculation (prec) of T (and Tr; NULL: self-join), the seeds QT(r H, j) of the rows
 *   r in [r_lo, r_hi) against every column j in [0, n), for every dimension, in the precalc's
 *   scaled units (x s_k, reading G16).  out: (r_hi - r_lo) x d x n doubles, [r][dim][j] (the half
 *   values the fused kernel would read).  scale_out: d doubles, the per-dimension scale of T
 *   (of Tr: multiply by Tr's scale, returned in scale_out[d .. 2d) for an AB-join). */
mp_status mp_selftest_seeds(mp_ctx* ctx, const double* T, const double* Tr, int64_t d, int64_t n, int64_t m,
                            mp_precision prec, int64_t H, int64_t r_lo, int64_t r_hi, double* out,
                            double* scale_out);
mp_status mp_selftest_precompute(mp_ctx* ctx, const double* T, int64_t d, int64_t n, int64_t m,
                                 mp_precision prec, double* df, double* dg, double* a);

#ifdef __cplusplus
}
#endif
#endif /* MP_H_ */

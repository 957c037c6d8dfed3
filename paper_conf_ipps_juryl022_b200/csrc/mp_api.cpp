// mp_api.cpp -- the C ABI (include/mp.h) and the host-side scheduler.
//
// Host responsibilities (the paper's Pseudocode 2 host driver, PAPER.md:L717-741,
// re-designed): argument validation, the fixed tile plan (diagonal blocks x H-row
// segments), the equal-cell diagonal-band partition across ranks (replaces the
// paper's round-robin tile assignment, L709-712), device scratch caching, and the
// launch sequence precompute -> fused diagonal kernel -> finalize.  All arithmetic of
// the method runs in the CUDA kernels (mp_kernels.cu); nothing here computes on data.
#include "../../include/mp.h"
#include "mp_internal.h"

#include <cuda.h>           // driver-API types only (VMM entry points are fetched at run time)
#include <cuda_fp16.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <string>
#include <vector>

namespace {

constexpr int64_t kDefaultH[6] = {4096, 1024, 256, 256, 256, 256};  // FP64, FP32, FP16, MIXED, FP16C, FP16CK (upper bounds)

// Default re-seed interval H (= tile height, the paper's tiling lever against error growth,
// PAPER.md:L700-703).  The recurrence error grows with H relative to the window energy, which
// scales with m, so reduced precisions re-seed every 8m rows (seed cost m/H stays 1/8 of a
// cell-dim's recurrence work), capped by the per-precision maximum.
int64_t default_h(int prec, int64_t m) {
    if (prec == MP_FP64) return kDefaultH[prec];
    return std::max<int64_t>(64, std::min<int64_t>(kDefaultH[prec], 8 * m));
}

struct Buf {
    void* p = nullptr;
    size_t bytes = 0;
};

}  // namespace

struct mp_ctx {
    int device = 0;
    int nsm = 148;
    cudaStream_t stream = nullptr;
    int64_t H[6] = {0, 0, 0, 0, 0, 0};
    std::string err;
    // cached scratch
    Buf dT, dTr, st_q, st_r, tw_q, tw_r, mu_q, mu_r, mup_q, mup_r, nrm, keys, ext, seg, counter, dP, dI, flag;
    Buf stp_q, stp_r, scale, scale_r, maxbits, flat;  // FP16 / Mixed precompute
    Buf seedtab;            // tensor-core seed table (seed_mode MP_SEEDS_TC)
    int seed_mode = MP_SEEDS_DIRECT;
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    int* hflag = nullptr;   // pinned read-back of the non-finite flag
    double last_ms = 0.0;
    int64_t last_launches = 0;
    // last mp_compute_stream: chunk geometry and peak physically mapped device bytes
    int64_t stream_R = 0, stream_Wb = 0, stream_peak = 0, stream_launches = 0;
    bool stream_timed = false;   // last_ms is the sum over the streamed launches
};

namespace {

mp_status fail(mp_ctx* ctx, mp_status st, const std::string& msg) {
    if (ctx) ctx->err = msg;
    return st;
}

mp_status cuda_fail(mp_ctx* ctx, cudaError_t e, const char* where) {
    return fail(ctx, e == cudaErrorMemoryAllocation ? MP_ERR_NOMEM : MP_ERR_CUDA,
                std::string(where) + ": " + cudaGetErrorString(e));
}

#define MP_CUDA(ctx, call)                                              \
    do {                                                                \
        cudaError_t e_ = (call);                                        \
        if (e_ != cudaSuccess) return cuda_fail((ctx), e_, #call);      \
    } while (0)

cudaError_t ensure(Buf& b, size_t bytes) {
    if (b.bytes >= bytes && b.p) return cudaSuccess;
    if (b.p) cudaFree(b.p);
    b.p = nullptr;
    b.bytes = 0;
    if (bytes == 0) bytes = 16;
    cudaError_t e = cudaMalloc(&b.p, bytes);
    if (e == cudaSuccess) b.bytes = bytes;
    return e;
}

void release(Buf& b) {
    if (b.p) cudaFree(b.p);
    b.p = nullptr;
    b.bytes = 0;
}

size_t elt_bytes(int prec) { return prec == MP_FP64 ? 8 : 4; }

// precompute over the whole series (every position resident)
void full_window(mpk::PreParams& pp, int64_t n, int64_t L) {
    pp.w0 = 0; pp.w1 = n; pp.T_off = 0; pp.T_ld = L; pp.s_off = 0; pp.s_end = n; pp.s_ld = n;
}

// ---------------------------------------------------------------- tile plan
struct Plan {
    int64_t dlo = 0, dhi = -1, nb = 0;
    int nc = 32, H = 1024;
    std::vector<long long> seg;    // nb + 1 exclusive prefix of segments
    std::vector<double> cells;     // nb + 1 exclusive prefix of cells
};

// Tile height: a multiple of the re-seed interval H (re-seeds inside a tile happen at
// warp-uniform steps, so taller tiles only amortise the per-tile stagger ramp), at most 4096
// rows, and short enough to leave >= ~20k tiles for the persistent warps.
#ifndef MP_TILE_MAX
#define MP_TILE_MAX 4096
#endif
#ifndef MP_TILE_GROW_BELOW
#define MP_TILE_GROW_BELOW 4096
#endif
int64_t tile_height(int64_t Hs, int64_t n, int64_t ndiag) {
    int64_t H = Hs;
    while (H < MP_TILE_GROW_BELOW && H * 2 <= MP_TILE_MAX && (double)ndiag * n / (H * 2) / 2.0 >= 20000.0) H *= 2;
    return H;
}

Plan build_plan(int64_t d, int64_t n, int64_t excl, bool self, int prec, int64_t Hs) {
    Plan pl;
    pl.nc = mpk::pick_variant(prec, (int)d).NC;
    const int64_t ndiag = self ? std::max<int64_t>(0, n - 1 - excl) : 2 * n - 1;
    const int64_t H = tile_height(Hs, n, ndiag);
    pl.H = (int)H;
    if (self) { pl.dlo = excl + 1; pl.dhi = n - 1; }
    else { pl.dlo = -(n - 1); pl.dhi = n - 1; }
    if (pl.dlo > pl.dhi) { pl.nb = 0; pl.seg.assign(1, 0); pl.cells.assign(1, 0.0); return pl; }
    pl.nb = (pl.dhi - pl.dlo + 1 + pl.nc - 1) / pl.nc;
    pl.seg.resize(pl.nb + 1);
    pl.cells.resize(pl.nb + 1);
    pl.seg[0] = 0;
    pl.cells[0] = 0;
    for (int64_t b = 0; b < pl.nb; ++b) {
        const int64_t d0 = pl.dlo + b * pl.nc, d1 = std::min(d0 + pl.nc - 1, pl.dhi);
        const int64_t rlo = std::max<int64_t>(0, -d1), rhi = std::min<int64_t>(n, n - std::max<int64_t>(d0, 0));
        int64_t nseg = 0;
        if (rlo < rhi) nseg = (rhi + H - 1) / H - rlo / H;
        double c = 0;
        for (int64_t dd = d0; dd <= d1; ++dd) c += (double)(n - (dd < 0 ? -dd : dd));
        pl.seg[b + 1] = pl.seg[b] + nseg;
        pl.cells[b + 1] = pl.cells[b] + c;
    }
    return pl;
}

// band g of world: blocks [bb[g], bb[g+1]) with (close to) equal cell counts
std::vector<int64_t> band_blocks(const Plan& pl, int world) {
    std::vector<int64_t> bb(world + 1, 0);
    const double tot = pl.cells[pl.nb];
    for (int g = 1; g < world; ++g) {
        const double target = tot * g / world;
        int64_t b = std::lower_bound(pl.cells.begin(), pl.cells.end(), target) - pl.cells.begin();
        bb[g] = std::min<int64_t>(std::max<int64_t>(b, bb[g - 1]), pl.nb);
    }
    bb[world] = pl.nb;
    return bb;
}

mp_status validate(mp_ctx* ctx, const void* T, int64_t d, int64_t n, int64_t m, int prec) {
    if (!T) return fail(ctx, MP_ERR_INVALID, "T is NULL");
    if (d < 1 || d > MP_MAX_D) return fail(ctx, MP_ERR_INVALID, "d must be in [1, 1024]");
    if (n < 2) return fail(ctx, MP_ERR_INVALID, "n must be >= 2");
    if (m < 2) return fail(ctx, MP_ERR_INVALID, "m must be >= 2");
    if (n >= (int64_t(1) << 31) - 1) return fail(ctx, MP_ERR_INVALID, "n must be < 2^31");
    if (m > (int64_t(1) << 20)) return fail(ctx, MP_ERR_INVALID, "m too large");
    if (prec < 0 || prec > 5) return fail(ctx, MP_ERR_INVALID, "unknown precision");
    if (prec == MP_FP64 && d > 512) return fail(ctx, MP_ERR_UNSUPPORTED, "FP64 supports d <= 512");
    return MP_OK;
}

// Launch the fused kernel over the tiles of diagonal blocks [B0, B1) of plan pl restricted to the
// row segments [q0, q1) (a whole band: q0 = 0, q1 = nq).  The band's blocks are renumbered from 0
// (delta_lo = the band's first diagonal), so every tile -- diagonal block x row segment, seeds at
// the segment start and at the fixed re-seed rows -- is the same computation as in the full plan:
// results do not depend on how the plan is cut into launches (ranks, streamed chunks).
// mp carries the data pointers and n, d, m, H; the tile fields are filled here.
mp_status enqueue_tiles(mp_ctx* ctx, cudaStream_t s, int prec, bool self, mpk::MainParams mp, const Plan& pl,
                        int64_t B0, int64_t B1, int64_t q0, int64_t q1, bool timed, Buf* pinned = nullptr) {
    const int64_t n = mp.n, HT = pl.H, NC = pl.nc, nb = B1 - B0;
    if (nb <= 0 || q1 <= q0) return MP_OK;
    const int64_t dlo = pl.dlo + B0 * NC, dhi = std::min<int64_t>(pl.dlo + B1 * NC - 1, pl.dhi);
    const int64_t nq = std::max<int64_t>(1, (n + HT - 1) / HT);
    // segments [qlo(b), qhi(b)) of band block b inside [q0, q1); both are non-increasing in b
    auto qlo = [&](int64_t b) {
        const int64_t d1 = std::min(dlo + b * NC + NC - 1, dhi);
        return std::max<int64_t>(q0, std::max<int64_t>(0, -d1) / HT);
    };
    auto qhi = [&](int64_t b) {
        const int64_t d0 = dlo + b * NC;
        return std::min<int64_t>(q1, (std::min<int64_t>(n, n - std::max<int64_t>(d0, 0)) + HT - 1) / HT);
    };
    auto first_b = [&](auto pred) {  // first b in [0, nb) with pred(b) (monotone), else nb
        int64_t lo = 0, hi = nb;
        while (lo < hi) {
            const int64_t mid = (lo + hi) / 2;
            if (pred(mid)) hi = mid; else lo = mid + 1;
        }
        return lo;
    };
    // [q_prefix (nq + 1) | q_block0 (nq) | seg_prefix (nb + 1)]
    std::vector<long long> tab(2 * nq + 1 + nb + 1);
    tab[0] = 0;
    for (int64_t q = 0; q < nq; ++q) {  // segment-major order (warp-tile kernels)
        const int64_t bs = first_b([&](int64_t b) { return qlo(b) <= q; });
        const int64_t be = first_b([&](int64_t b) { return qhi(b) <= q; });
        tab[q + 1] = tab[q] + std::max<int64_t>(0, be - bs);
        tab[nq + 1 + q] = bs;
    }
    long long* segp = tab.data() + 2 * nq + 1;   // block-major order (block-cooperative kernels)
    segp[0] = 0;
    for (int64_t b = 0; b < nb; ++b) segp[b + 1] = segp[b] + std::max<int64_t>(0, qhi(b) - qlo(b));
    const long long total = segp[nb];
    if (tab[nq] != total) return fail(ctx, MP_ERR_INVALID, "internal: tile plan mismatch");
    if (total == 0) return MP_OK;
    MP_CUDA(ctx, ensure(ctx->seg, tab.size() * sizeof(long long)));
    const void* src = tab.data();
    if (pinned) {   // a pinned copy: the upload is then asynchronous (a pageable one waits for the stream)
        if (pinned->bytes < tab.size() * sizeof(long long)) {
            if (pinned->p) cudaFreeHost(pinned->p);
            pinned->p = nullptr;
            pinned->bytes = 0;
            MP_CUDA(ctx, cudaHostAlloc(&pinned->p, tab.size() * sizeof(long long) * 2, cudaHostAllocDefault));
            pinned->bytes = tab.size() * sizeof(long long) * 2;
        }
        std::memcpy(pinned->p, tab.data(), tab.size() * sizeof(long long));
        src = pinned->p;
    }
    MP_CUDA(ctx, cudaMemcpyAsync(ctx->seg.p, src, tab.size() * sizeof(long long), cudaMemcpyHostToDevice, s));
    MP_CUDA(ctx, ensure(ctx->counter, sizeof(unsigned long long)));
    MP_CUDA(ctx, cudaMemsetAsync(ctx->counter.p, 0, sizeof(unsigned long long), s));
    const mpk::Variant var = mpk::pick_variant(prec, mp.d);
    mp.order = var.cta ? 0 : 1;   // decode_tile (mp_diag.cuh) says why
    mp.q_prefix = (const long long*)ctx->seg.p;
    mp.q_block0 = (const long long*)ctx->seg.p + nq + 1;
    mp.nq = nq;
    mp.seg_prefix = (const long long*)ctx->seg.p + 2 * nq + 1;
    mp.nb = nb;
    mp.t_begin = 0;
    mp.t_count = total;
    mp.counter = (unsigned long long*)ctx->counter.p;
    mp.HT = pl.H;
    mp.delta_lo = dlo; mp.delta_hi = dhi;
    mp.q_lo = q0;
    const int bps = std::max(1, mpk::main_blocks_per_sm(prec, mp.d, self));
    long long grid = (long long)ctx->nsm * bps;
    const int wpb = std::max(1, mpk::variant_warps_per_block(prec, mp.d, self));
    grid = std::min<long long>(grid, (total + wpb - 1) / wpb);
    grid = std::max<long long>(grid, 1);
    if (timed) MP_CUDA(ctx, cudaEventRecord(ctx->ev0, s));
    MP_CUDA(ctx, mpk::launch_main(prec, self, mp, (int)grid, s));
    if (timed) MP_CUDA(ctx, cudaEventRecord(ctx->ev1, s));
    ctx->last_launches += 1;
    return MP_OK;
}

// FP32 windows shorter than kCompMinM run the plain QT recurrence in the warp kernels (P32N): the
// compensated one (reading R4) is needed for the 1e-4 gate at m >= 256 only
// (C2 FP32: 45.4 -> 44.4 ms without it).  The block kernels (d >= 64) always compensate.
constexpr int64_t kCompMinM = 192;
int kernel_prec(int prec, int64_t m, const mpk::Variant& var) {
    return (prec == MP_FP32 && m < kCompMinM && !var.cta && !var.ctab) ? (int)mpk::P32N : prec;
}

// Tensor-core seeds apply to the FP32-precalc half modes (Mixed, FP16CK) on the block kernels.
// seed table per row chunk (device bytes): up to 128 seed rows (one MMA tile of M = 128) per chunk,
// so each Hankel operand tile the GEMM builds serves as many rows as fit
constexpr int64_t kSeedTabBytes = int64_t(8) << 30;
bool tc_seeds(const mp_ctx* ctx, int prec) {
    return ctx->seed_mode == MP_SEEDS_TC && (prec == MP_MIXED || prec == MP_FP16CK);
}

// Re-seed interval of a run: the context's (mp_config.reseed_h) or the default, rounded up to a
// multiple of 8 (every kernel steps in batches of 1, 2 or 4 rows, so every re-seed row
// i = 0 mod H is a batch start in every kernel variant; include/mp.h, mp_config.reseed_h).
int64_t reseed_interval(const mp_ctx* ctx, int prec, int64_t m) {
    const int64_t H = ctx->H[prec] > 0 ? ctx->H[prec] : default_h(prec, m);
    return std::min<int64_t>((H + 7) / 8 * 8, int64_t(1) << 30);
}

// Device pipeline: keys for band (rank, world) of the tile plan, internal key format.
mp_status run_partial(mp_ctx* ctx, cudaStream_t s, const double* dT, const double* dTr, int64_t d,
                      int64_t n, int64_t m, int prec, int64_t excl, int rank, int world, bool pre_only = false) {
    const bool self = dTr == nullptr;
    const int64_t L = n + m - 1;
    const size_t eb = elt_bytes(prec);
    // re-seeds happen at staging-batch starts (every kernel steps in batches of 1, 2 or 4 rows),
    // so the interval is rounded up to a multiple of 8: then every re-seed row i = 0 mod H is a
    // batch start in every kernel variant (include/mp.h, mp_config.reseed_h)
    const int64_t H = reseed_interval(ctx, prec, m);
    ctx->stream_timed = false;
    if (self && excl < 0) excl = (m + 3) / 4;

    // flag non-finite inputs (reading G23).  The flag is read back after the whole pipeline is
    // enqueued (finish_partial), so the check costs one O(d L) kernel and no mid-pipeline host
    // sync; a non-finite input only makes the kernels compute NaN distances, which never pass
    // a profile update, before the call reports MP_ERR_INVALID.
    MP_CUDA(ctx, ensure(ctx->flag, sizeof(int)));
    MP_CUDA(ctx, cudaMemsetAsync(ctx->flag.p, 0, sizeof(int), s));
    MP_CUDA(ctx, mpk::launch_check_finite(dT, d * L, (int*)ctx->flag.p, s));
    if (!self) MP_CUDA(ctx, mpk::launch_check_finite(dTr, d * L, (int*)ctx->flag.p, s));

    // precalculation (Pseudocode 1 line 2)
    const bool half = prec == MP_FP16 || prec == MP_MIXED || prec == MP_FP16C || prec == MP_FP16CK;
    const size_t sb = half ? 16 : 4 * eb;                                   // stats entry bytes
    const size_t tb = prec == MP_FP64 ? 8 : ((prec == MP_FP16 || prec == MP_FP16C) ? 2 : 4);  // precalc value bytes
    const size_t tbs = prec == MP_FP32 ? 8 : tb;  // window stats scratch (FP32 mode: FP64 precalc, reading R1')
    const mpk::Variant var = mpk::pick_variant(prec, (int)d);
    const int Dp = var.DL * var.G;
    mpk::PreParams pp{};
    pp.n = n; pp.d = (int)d; pp.m = (int)m; pp.Dp = Dp;
    full_window(pp, n, L);
    if (var.ctab) { pp.pm_G = var.G; pp.pm_DL = var.DL; }
    MP_CUDA(ctx, ensure(ctx->nrm, (size_t)n * d * tbs));
    pp.nrm32 = (float*)ctx->nrm.p; pp.nrm64 = (double*)ctx->nrm.p;
    if (half) {
        MP_CUDA(ctx, ensure(ctx->scale, (size_t)d * sizeof(double)));
        MP_CUDA(ctx, ensure(ctx->scale_r, (size_t)d * sizeof(double)));
        MP_CUDA(ctx, ensure(ctx->maxbits, (size_t)d * 2 * sizeof(unsigned long long)));
        MP_CUDA(ctx, ensure(ctx->flat, (size_t)n * d * 3 * 2));
        pp.scale = (double*)ctx->scale.p; pp.maxbits = (unsigned long long*)ctx->maxbits.p; pp.flat = ctx->flat.p;
    }
    Buf* series_bufs[2][5] = {{&ctx->st_q, &ctx->stp_q, &ctx->mu_q, &ctx->mup_q, &ctx->tw_q},
                              {&ctx->st_r, &ctx->stp_r, &ctx->mu_r, &ctx->mup_r, &ctx->tw_r}};
    for (int sidx = 0; sidx < (self ? 1 : 2); ++sidx) {
        Buf** B = series_bufs[sidx];
        MP_CUDA(ctx, ensure(*B[0], (size_t)n * d * sb));
        if (half) MP_CUDA(ctx, ensure(*B[1], (size_t)(n + 1) * d * sb));  // pair format: n+1 entries
        MP_CUDA(ctx, ensure(*B[2], (size_t)n * d * tbs));
        MP_CUDA(ctx, ensure(*B[3], (size_t)n * Dp * tb));
        MP_CUDA(ctx, ensure(*B[4], (size_t)L * Dp * tb));
        pp.T = sidx == 0 ? dT : dTr;
        if (half) pp.scale = (double*)(sidx == 0 ? ctx->scale.p : ctx->scale_r.p);   // one scale per series
        pp.st = B[0]->p; pp.st_pair = B[1]->p; pp.mu = B[2]->p; pp.mup = B[3]->p; pp.tw = B[4]->p;
        MP_CUDA(ctx, mpk::launch_precompute(prec, pp, s));
    }
    if (pre_only) return MP_OK;   // mp_selftest_seeds

    // keys (FP16 / Mixed use the FP32 key format: float bits of the half-precision sum)
    const size_t kb = (size_t)n * d * (prec == MP_FP64 ? 16 : 8);
    MP_CUDA(ctx, ensure(ctx->keys, kb + 16));   // + 16: TMA key rows are 16-byte aligned supersets
    MP_CUDA(ctx, mpk::launch_init_keys(prec, ctx->keys.p, n * d, s));

    // plan + band
    Plan pl = build_plan(d, n, excl, self, prec, H);
    ctx->last_launches = 0;
    ctx->last_ms = 0.0;
    if (pl.nb > 0) {
        std::vector<int64_t> bb = band_blocks(pl, world);
        mpk::MainParams mp{};
        mp.st_q = ctx->st_q.p;
        mp.st_r = self ? ctx->st_q.p : ctx->st_r.p;
        if (half) mp.st_r = self ? ctx->stp_q.p : ctx->stp_r.p;   // columns: pair format
        mp.tw_q = ctx->tw_q.p;
        mp.tw_r = self ? ctx->tw_q.p : ctx->tw_r.p;
        mp.mu_q = ctx->mup_q.p;
        mp.mu_r = self ? ctx->mup_q.p : ctx->mup_r.p;
        mp.keys = ctx->keys.p;
        mp.n = n; mp.d = (int)d; mp.m = (int)m; mp.H = (int)H;
        const int64_t nq = std::max<int64_t>(1, (n + pl.H - 1) / pl.H);
        if (!(tc_seeds(ctx, prec) && var.cta))
            return enqueue_tiles(ctx, s, kernel_prec(prec, m, var), self, mp, pl, bb[rank], bb[rank + 1], 0, nq, true);
        // tensor-core seeds (NEXT-3): per row chunk, one seed GEMM for the chunk's re-seed rows,
        // then the fused kernel over the chunk's tiles reading the table
        const int64_t B0 = bb[rank], B1 = bb[rank + 1];
        if (B1 <= B0) return MP_OK;
        const int64_t dlo = pl.dlo + B0 * pl.nc, dhi = std::min<int64_t>(pl.dlo + B1 * pl.nc - 1, pl.dhi);
        const int64_t ncol = n + 8;
        const int64_t rows_seg = std::max<int64_t>(1, pl.H / H);              // seed rows per row segment
        const int64_t per_seg = rows_seg * d * ncol * 2;                       // table bytes per row segment
        const int64_t qs = std::max<int64_t>(1, std::min(kSeedTabBytes / per_seg, std::max<int64_t>(1, 128 / rows_seg)));
        MP_CUDA(ctx, ensure(ctx->seedtab, (size_t)(qs * per_seg + 64)));
        mpk::SeedParams sp{};
        sp.Tq = dT; sp.Tr = self ? dT : dTr;
        sp.scale_q = (const double*)ctx->scale.p;
        sp.scale_r = (const double*)(self ? ctx->scale.p : ctx->scale_r.p);
        sp.mu_q = (const float*)ctx->mu_q.p;
        sp.mu_r = (const float*)(self ? ctx->mu_q.p : ctx->mu_r.p);
        sp.tab = ctx->seedtab.p;
        sp.n = n; sp.d = (int)d; sp.m = (int)m; sp.H = (int)H;
        MP_CUDA(ctx, cudaEventRecord(ctx->ev0, s));
        for (int64_t q0 = 0; q0 < nq; q0 += qs) {
            const int64_t q1 = std::min(nq, q0 + qs), i0 = q0 * pl.H, i1 = std::min(n, q1 * pl.H);
            sp.r_lo = (i0 + H - 1) / H;
            sp.r_hi = (i1 + H - 1) / H;
            sp.j_lo = std::max<int64_t>(0, i0 + dlo) / 8 * 8;
            sp.j_hi = std::min<int64_t>(n, std::max<int64_t>(0, i1 - 1 + dhi + 1));
            if (sp.j_hi <= sp.j_lo) continue;
            sp.ldj = (sp.j_hi - sp.j_lo + 7) / 8 * 8;
            MP_CUDA(ctx, mpk::launch_seed_gemm(sp, s));
            mp.seed_tab = sp.tab;
            mp.tab_r_lo = sp.r_lo; mp.tab_r_hi = sp.r_hi; mp.tab_j_lo = sp.j_lo; mp.tab_ldj = sp.ldj;
            mp_status st2 = enqueue_tiles(ctx, s, prec, self, mp, pl, B0, B1, q0, q1, false);
            if (st2 != MP_OK) return st2;
        }
        MP_CUDA(ctx, cudaEventRecord(ctx->ev1, s));
    }
    return MP_OK;
}

// Read back the non-finite flag of the last run_partial (after the caller's remaining work on
// stream s is enqueued): one pinned 4-byte copy and a stream sync.
mp_status finish_partial(mp_ctx* ctx, cudaStream_t s) {
    if (!ctx->hflag) MP_CUDA(ctx, cudaHostAlloc((void**)&ctx->hflag, sizeof(int), cudaHostAllocDefault));
    MP_CUDA(ctx, cudaMemcpyAsync(ctx->hflag, ctx->flag.p, sizeof(int), cudaMemcpyDeviceToHost, s));
    MP_CUDA(ctx, cudaStreamSynchronize(s));
    if (*ctx->hflag) return fail(ctx, MP_ERR_INVALID, "non-finite input");
    return MP_OK;
}


// ---------------------------------------------------------------- beyond-memory streaming (NEXT-4)
// PAPER.md:L693-699 (the tiling "decouples the size of the distance matrix ... despite the
// limited device memory") and L2432-2433; SURVEY 8(f) NEXT-4.  The host keeps T, Tr and the
// running merge keys; the device holds, per step, the statistics / seed operands / keys of one
// row window [i0, i1) and one column window (the columns of a diagonal band over those rows).
// Every device array keeps its absolute-position layout inside a virtual-address reservation of
// the full size (CUDA VMM): only the granules of the current windows are backed by physical
// memory, so the fused kernels run unchanged, and a position outside the windows would fault.

typedef CUresult (*PF_memCreate)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*, unsigned long long);
typedef CUresult (*PF_memRelease)(CUmemGenericAllocationHandle);
typedef CUresult (*PF_addrReserve)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long);
typedef CUresult (*PF_addrFree)(CUdeviceptr, size_t);
typedef CUresult (*PF_memMap)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long);
typedef CUresult (*PF_memUnmap)(CUdeviceptr, size_t);
typedef CUresult (*PF_memSetAccess)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t);
typedef CUresult (*PF_memGran)(size_t*, const CUmemAllocationProp*, CUmemAllocationGranularity_flags);

struct VArr {                                      // one virtual array
    const char* name = "";
    CUdeviceptr base = 0;
    size_t bytes = 0;                              // reserved (a multiple of the granularity)
    std::vector<CUmemGenericAllocationHandle> h;   // per granule, 0 = unmapped
    std::vector<char> saved;                       // keys: the granule's bytes live in the host store
    void* ptr() const { return (void*)base; }
};

struct Vmm {
    PF_memCreate create = nullptr; PF_memRelease release = nullptr; PF_addrReserve reserve = nullptr;
    PF_addrFree afree = nullptr; PF_memMap map = nullptr; PF_memUnmap unmap = nullptr;
    PF_memSetAccess access = nullptr; PF_memGran granularity = nullptr;
    CUmemAllocationProp prop{};
    CUmemAccessDesc acc{};
    size_t gran = 0, mapped = 0, peak = 0;
    std::vector<CUmemGenericAllocationHandle> pool;   // unmapped physical granules, reused
    std::vector<VArr*> arrs;

    std::string load(int dev) {
        auto get = [](const char* name, void** fp) {
            cudaDriverEntryPointQueryResult q;
            return cudaGetDriverEntryPoint(name, fp, cudaEnableDefault, &q) == cudaSuccess &&
                   q == cudaDriverEntryPointSuccess && *fp != nullptr;
        };
        if (!get("cuMemCreate", (void**)&create) || !get("cuMemRelease", (void**)&release) ||
            !get("cuMemAddressReserve", (void**)&reserve) || !get("cuMemAddressFree", (void**)&afree) ||
            !get("cuMemMap", (void**)&map) || !get("cuMemUnmap", (void**)&unmap) ||
            !get("cuMemSetAccess", (void**)&access) || !get("cuMemGetAllocationGranularity", (void**)&granularity))
            return "CUDA driver VMM entry points unavailable";
        prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
        prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
        prop.location.id = dev;
        acc.location = prop.location;
        acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
        if (granularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS || gran == 0)
            return "cuMemGetAllocationGranularity failed";
        return "";
    }
    CUresult reserve_arr(VArr& a, size_t bytes) {
        a.bytes = std::max<size_t>(gran, (bytes + gran - 1) / gran * gran);
        CUresult r = reserve(&a.base, a.bytes, gran, 0, 0);
        if (r != CUDA_SUCCESS) { a.base = 0; return r; }
        a.h.assign(a.bytes / gran, 0);
        a.saved.assign(a.bytes / gran, 0);
        arrs.push_back(&a);
        return CUDA_SUCCESS;
    }
    // map granule g (its access rights are set per contiguous run by set_access)
    CUresult map_g(VArr& a, size_t g) {
        CUmemGenericAllocationHandle hd = 0;
        if (!pool.empty()) { hd = pool.back(); pool.pop_back(); }
        else { CUresult r = create(&hd, gran, &prop, 0); if (r != CUDA_SUCCESS) return r; }
        CUresult r = map(a.base + g * gran, gran, 0, hd, 0);
        if (r != CUDA_SUCCESS) { pool.push_back(hd); return r; }
        a.h[g] = hd;
        mapped += gran;
        peak = std::max(peak, mapped);
        return CUDA_SUCCESS;
    }
    CUresult set_access(VArr& a, size_t g0, size_t g1) { return access(a.base + g0 * gran, (g1 - g0) * gran, &acc, 1); }
    // unmap granules [g0, g1) (each mapped separately) with one call; per granule if the driver
    // refuses a range spanning several mappings
    CUresult unmap_run(VArr& a, size_t g0, size_t g1) {
        if (g1 - g0 > 1 && multi_unmap) {
            if (unmap(a.base + g0 * gran, (g1 - g0) * gran) == CUDA_SUCCESS) {
                for (size_t g = g0; g < g1; ++g) { pool.push_back(a.h[g]); a.h[g] = 0; mapped -= gran; }
                return CUDA_SUCCESS;
            }
            multi_unmap = false;
        }
        for (size_t g = g0; g < g1; ++g) {
            CUresult r = unmap_g(a, g);
            if (r != CUDA_SUCCESS) return r;
        }
        return CUDA_SUCCESS;
    }
    bool multi_unmap = true;
    CUresult unmap_g(VArr& a, size_t g) {
        CUresult r = unmap(a.base + g * gran, gran);
        pool.push_back(a.h[g]);
        a.h[g] = 0;
        mapped -= gran;
        return r;
    }
    void destroy() {
        for (VArr* a : arrs) {
            for (size_t g = 0; g < a->h.size(); ++g) if (a->h[g]) unmap_g(*a, g);
            if (a->base) afree(a->base, a->bytes);
            a->base = 0;
        }
        arrs.clear();
        for (auto hd : pool) release(hd);
        pool.clear();
    }
};

using Ivl = std::pair<int64_t, int64_t>;   // position interval [first, second)

std::vector<Ivl> merge_ivls(std::vector<Ivl> v) {
    std::vector<Ivl> o;
    std::sort(v.begin(), v.end());
    for (const Ivl& x : v) {
        if (x.first >= x.second) continue;
        if (!o.empty() && x.first <= o.back().second) o.back().second = std::max(o.back().second, x.second);
        else o.push_back(x);
    }
    return o;
}
std::vector<Ivl> minus_ivls(const std::vector<Ivl>& a, const std::vector<Ivl>& b) {  // a \ b (both merged)
    std::vector<Ivl> o;
    for (Ivl x : a) {
        int64_t lo = x.first;
        for (const Ivl& y : b) {
            if (y.second <= lo || y.first >= x.second) continue;
            if (y.first > lo) o.push_back({lo, y.first});
            lo = std::max(lo, y.second);
        }
        if (lo < x.second) o.push_back({lo, x.second});
    }
    return o;
}

// Chunk geometry of a streamed run: rows per chunk R (a multiple of the tile height) and
// diagonals per band Wb (a multiple of the block width, Wb ~ 2R), the largest that fit the
// device budget (bytes per resident position x window sizes + fixed granule margins).
struct StreamGeo {
    int64_t R = 0, Wb = 0, HT = 0, NC = 0;
    double per_R = 0, fixed = 0;
    size_t sb = 0, tb = 0, tbs = 0, kb = 0;
    int Dp = 0;
    bool half = false;
};
mp_status plan_stream(mp_ctx* ctx, int64_t d, int64_t n, int64_t m, int prec, int64_t excl, bool self,
                      int64_t budget, size_t gran, const Plan& pl, StreamGeo& g) {
    const mpk::Variant var = mpk::pick_variant(prec, (int)d);
    g.half = prec == MP_FP16 || prec == MP_MIXED || prec == MP_FP16C || prec == MP_FP16CK;
    g.sb = g.half ? 8 : 4 * elt_bytes(prec);   // stats entry bytes (half: the row format RH, 4 halves)
    g.tb = prec == MP_FP64 ? 8 : ((prec == MP_FP16 || prec == MP_FP16C) ? 2 : 4);
    g.tbs = prec == MP_FP32 ? 8 : g.tb;
    g.kb = prec == MP_FP64 ? 16 : 8;
    g.Dp = var.DL * var.G;
    g.HT = pl.H;
    g.NC = pl.nc;
    const double side = (double)d * g.sb + (g.half ? d * 16.0 : 0.0) + 2.0 * g.Dp * g.tb;   // st, stp, tw, mup
    const double key = (double)d * g.kb;
    const double scr = (double)d * (2.0 * g.tbs + (g.half ? 6.0 : 0.0) + 8.0);             // mu, nrm, flat, T slice
    const double out = 16.0 * d;                                                            // P, I row window
    // windows of two consecutive steps are resident (the next step is prepared while the current
    // kernel runs): rows R, columns of two bands R + 2 Wb = 5R (Wb = 2R)
    g.per_R = self ? 6.0 * (side + key) + 3.0 * scr + out : (side + key) + 5.0 * side + 3.0 * scr + out;
    const int narr = g.half ? 5 : 4;   // st, (stp), tw, mup, keys per side
    g.fixed = (double)gran * 2.0 /* windows */ * 2.0 /* partial granules */ * narr * (self ? 1 : 2) +
              2.0 * m * g.Dp * g.tb + 6.0 * scr + (16 << 20);
    const double avail = (double)budget - g.fixed;
    int64_t R = avail > 0 ? (int64_t)(avail / g.per_R) : 0;
    R = R / g.HT * g.HT;
    if (R < g.HT)
        return fail(ctx, MP_ERR_NOMEM, "device budget too small for one row segment of the tile plan");
    R = std::min<int64_t>(R, (n + g.HT - 1) / g.HT * g.HT);
    g.R = R;
    g.Wb = std::max<int64_t>(g.NC, (2 * R) / g.NC * g.NC);
    (void)excl;
    return MP_OK;
}

struct Side {
    VArr st, stp, tw, mup, keys;
    std::vector<Ivl> valid;   // positions whose precompute is resident
    Buf scale;
    const double* T = nullptr;
};

#define MP_CU(ctx, call)                                                                        \
    do {                                                                                        \
        CUresult r_ = (call);                                                                   \
        if (r_ != CUDA_SUCCESS)                                                                 \
            return fail((ctx), r_ == CUDA_ERROR_OUT_OF_MEMORY ? MP_ERR_NOMEM : MP_ERR_CUDA,     \
                        std::string(#call) + ": CUresult " + std::to_string((int)r_));          \
    } while (0)

struct Streamer {
    // MP_STREAM_PROFILE=1: host seconds per phase, printed to stderr at the end of the call
    double t_sync = 0, t_remap = 0, t_pre = 0, t_fin = 0, t_save = 0, t_unmap = 0, t_map = 0;
    static double now() {
        return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
    }
    mp_ctx* ctx;
    cudaStream_t s;
    Vmm vm;
    StreamGeo g;
    int prec;
    int64_t d, n, m, L;
    bool self;
    unsigned char* hkeys = nullptr;        // host key store (pinned), absolute byte layout
    bool own_s = true;                     // S.s created here (destroyed at the end of the call)
    Buf tslice, mu, nrm, flat, maxbits, dPw, dIw;
    int64_t wmax = 0;
    Side sq, sr;

    // granules of array a covering the byte ranges of position intervals (+ trailing positions ex)
    std::vector<char> need_mask(const VArr& a, const std::vector<Ivl>& iv, double bpp, int64_t ex) const {
        std::vector<char> nm(a.h.size(), 0);
        for (const Ivl& x : iv) {
            const size_t lo = (size_t)(x.first * bpp), hi = std::min(a.bytes, (size_t)((x.second + ex) * bpp));
            if (hi <= lo) continue;
            for (size_t gi = lo / vm.gran; gi < (hi + vm.gran - 1) / vm.gran; ++gi) nm[gi] = 1;
        }
        return nm;
    }
    mp_status remap(VArr& a, const std::vector<char>& nm, bool is_keys, int64_t final_upto) {
        const double t0 = now();
        struct Acc { double& t; double t0; ~Acc() { t += now() - t0; } } acc{t_remap, t0};
        const size_t ng = a.h.size();
        if (is_keys) {   // save the key granules about to be unmapped (those still accumulating), per run
            bool any = false;
            for (size_t gi = 0; gi < ng;) {
                const bool sv = a.h[gi] && !nm[gi] && (int64_t)((gi * vm.gran + vm.gran - 1) / (d * g.kb)) >= final_upto;
                if (a.h[gi] && !nm[gi] && !sv) a.saved[gi] = 0;   // finalized rows: dropped
                if (!sv) { ++gi; continue; }
                size_t ge = gi;
                while (ge < ng && a.h[ge] && !nm[ge] && (int64_t)((ge * vm.gran + vm.gran - 1) / (d * g.kb)) >= final_upto)
                    a.saved[ge++] = 1;
                MP_CUDA(ctx, cudaMemcpyAsync(hkeys + gi * vm.gran, (char*)a.ptr() + gi * vm.gran, (ge - gi) * vm.gran,
                                             cudaMemcpyDeviceToHost, s));
                any = true;
                gi = ge;
            }
            if (any) MP_CUDA(ctx, cudaStreamSynchronize(s));
            t_save += now() - t0;
        }
        const double tu = now();
        static const char* keep_env = std::getenv("MP_STREAM_NOUNMAP");   // debugging knob: "1" or an array name
        const bool keep_all = keep_env && (std::strcmp(keep_env, "1") == 0 || std::strcmp(keep_env, a.name) == 0);
        for (size_t gi = 0; gi < ng && !keep_all;) {   // unmap the leaving granules, one call per run
            if (!(a.h[gi] && !nm[gi])) { ++gi; continue; }
            size_t ge = gi;
            while (ge < ng && a.h[ge] && !nm[ge]) ++ge;
            MP_CU(ctx, vm.unmap_run(a, gi, ge));
            gi = ge;
        }
        const double tm = now();
        t_unmap += tm - tu;
        struct AccM { double& t; double t0; ~AccM() { t += now() - t0; } } accm{t_map, tm};
        for (size_t gi = 0; gi < ng;) {   // map the new granules, one access call and copy per run
            if (a.h[gi] || !nm[gi]) { ++gi; continue; }
            size_t ge = gi;
            while (ge < ng && !a.h[ge] && nm[ge]) MP_CU(ctx, vm.map_g(a, ge++));
            MP_CU(ctx, vm.set_access(a, gi, ge));
            if (is_keys) {
                for (size_t k0 = gi; k0 < ge;) {
                    size_t k1 = k0;
                    while (k1 < ge && a.saved[k1] == a.saved[k0]) ++k1;
                    char* dptr = (char*)a.ptr() + k0 * vm.gran;
                    if (a.saved[k0]) MP_CUDA(ctx, cudaMemcpyAsync(dptr, hkeys + k0 * vm.gran, (k1 - k0) * vm.gran, cudaMemcpyHostToDevice, s));
                    else MP_CUDA(ctx, mpk::launch_init_keys(prec, dptr, (long long)((k1 - k0) * vm.gran / g.kb), s));
                    k0 = k1;
                }
            }
            gi = ge;
        }
        return MP_OK;
    }
    // precompute positions [a, b) of one series (statistics, pair format, seed operands)
    mp_status precompute(Side& sd, int64_t a, int64_t b) {
        struct Acc { double& t; double t0; ~Acc() { t += now() - t0; } } acc{t_pre, now()};
        mpk::PreParams pp{};
        pp.n = n; pp.d = (int)d; pp.m = (int)m; pp.Dp = g.Dp;
        const mpk::Variant var = mpk::pick_variant(prec, (int)d);
        if (var.ctab) { pp.pm_G = var.G; pp.pm_DL = var.DL; }
        pp.w0 = a; pp.w1 = b;
        pp.s_off = std::max<int64_t>(0, a - 2);
        pp.s_end = std::min<int64_t>(n, b + 1);
        pp.s_ld = pp.s_end - pp.s_off;
        pp.T_off = pp.s_off;
        const int64_t len = pp.s_end + m - 1 - pp.s_off;
        pp.T_ld = len;
        MP_CUDA(ctx, cudaMemcpy2DAsync(tslice.p, len * 8, sd.T + pp.s_off, L * 8, len * 8, d, cudaMemcpyHostToDevice, s));
        pp.T = (const double*)tslice.p;
        pp.st = sd.st.ptr(); pp.st_pair = sd.stp.ptr(); pp.tw = sd.tw.ptr(); pp.mup = sd.mup.ptr();
        pp.mu = mu.p; pp.nrm32 = (float*)nrm.p; pp.nrm64 = (double*)nrm.p; pp.flat = flat.p;
        pp.scale = (double*)sd.scale.p; pp.maxbits = (unsigned long long*)maxbits.p;
        MP_CUDA(ctx, mpk::launch_precompute(prec, pp, s, false));
        return MP_OK;
    }
    // non-finite input (reading G23) over the whole series, one window at a time
    mp_status check_pass(Side& sd) {
        for (int64_t a = 0; a < L; a += wmax) {
            const int64_t len = std::min(L, a + wmax) - a;
            MP_CUDA(ctx, cudaMemcpy2DAsync(tslice.p, len * 8, sd.T + a, L * 8, len * 8, d, cudaMemcpyHostToDevice, s));
            MP_CUDA(ctx, mpk::launch_check_finite((const double*)tslice.p, d * len, (int*)ctx->flag.p, s));
        }
        return MP_OK;
    }
    // per-dimension half-precision scale of one series over all its windows (reading G16)
    mp_status half_scale(Side& sd) {
        for (int64_t a = 0; a < n; a += wmax) {
            const int64_t b = std::min(n, a + wmax);
            mpk::PreParams pp{};
            pp.n = n; pp.d = (int)d; pp.m = (int)m;
            const int64_t len = b + m - 1 - a;
            pp.w0 = a; pp.w1 = b; pp.T_off = a; pp.T_ld = len;
            MP_CUDA(ctx, cudaMemcpy2DAsync(tslice.p, len * 8, sd.T + a, L * 8, len * 8, d, cudaMemcpyHostToDevice, s));
            pp.T = (const double*)tslice.p;
            pp.maxbits = (unsigned long long*)maxbits.p;
            pp.scale = (double*)sd.scale.p;
            MP_CUDA(ctx, mpk::launch_scale_max(pp, a == 0, s));
            if (b == n) MP_CUDA(ctx, mpk::launch_scale_pick(prec, pp, s));
        }
        return MP_OK;
    }
    // make the positions `iv` of one series resident (and its keys `kv`: query series only)
    mp_status ensure_side(Side& sd, std::vector<Ivl> iv, const std::vector<Ivl>* kv, int64_t final_upto) {
        iv = merge_ivls(iv);
        const double dd = (double)d;
        mp_status st;
        if ((st = remap(sd.st, need_mask(sd.st, iv, dd * g.sb, 0), false, 0)) != MP_OK) return st;
        if (g.half && (st = remap(sd.stp, need_mask(sd.stp, iv, dd * 16, 1), false, 0)) != MP_OK) return st;
        if ((st = remap(sd.tw, need_mask(sd.tw, iv, (double)g.Dp * g.tb, m - 1), false, 0)) != MP_OK) return st;
        if ((st = remap(sd.mup, need_mask(sd.mup, iv, (double)g.Dp * g.tb, 0), false, 0)) != MP_OK) return st;
        if (kv) {
            const std::vector<Ivl> kk = merge_ivls(*kv);
            if ((st = remap(sd.keys, need_mask(sd.keys, kk, dd * g.kb, 0), true, final_upto)) != MP_OK) return st;
        }
        const int64_t piece = wmax - 4;   // the window scratch holds R + Wb positions
        for (const Ivl& x : minus_ivls(iv, sd.valid))
            for (int64_t a = x.first; a < x.second; a += piece)
                if ((st = precompute(sd, a, std::min(x.second, a + piece))) != MP_OK) return st;
        sd.valid = iv;
        return MP_OK;
    }
};

constexpr int64_t kWinPad = 8;   // positions of margin around each streamed window

mp_status run_stream(mp_ctx* ctx, const double* T, const double* Tr, int64_t d, int64_t n, int64_t m, int prec,
                     int64_t excl, int64_t budget, double* P, int64_t* I) {
    const bool self = Tr == nullptr;
    if (self && excl < 0) excl = (m + 3) / 4;
    const int64_t L = n + m - 1;
    const int64_t H = reseed_interval(ctx, prec, m);
    const Plan pl = build_plan(d, n, excl, self, prec, H);
    Streamer S{};
    S.ctx = ctx;
    // S.s: the prep stream (remaps, key copies, window precompute); ctx->stream computes
    if (cudaStreamCreateWithFlags(&S.s, cudaStreamNonBlocking) != cudaSuccess) return fail(ctx, MP_ERR_CUDA, "stream");
    S.prec = prec; S.d = d; S.n = n; S.m = m; S.L = L; S.self = self;
    const std::string err = S.vm.load(ctx->device);
    if (!err.empty()) return fail(ctx, MP_ERR_UNSUPPORTED, err);
    mp_status st = plan_stream(ctx, d, n, m, prec, excl, self, budget, S.vm.gran, pl, S.g);
    if (st != MP_OK) return st;
    // testing knobs: force a finer geometry (rows rounded to the tile height, diagonals to the
    // block width) so small inputs exercise many chunks (include/mp.h)
    if (const char* e = std::getenv("MP_STREAM_ROWS")) {
        const int64_t r = std::max<int64_t>(1, std::atoll(e));
        S.g.R = std::max<int64_t>(S.g.HT, (r + S.g.HT - 1) / S.g.HT * S.g.HT);
    }
    if (const char* e = std::getenv("MP_STREAM_DIAGS")) {
        const int64_t w = std::max<int64_t>(1, std::atoll(e));
        S.g.Wb = std::max<int64_t>(S.g.NC, (w + S.g.NC - 1) / S.g.NC * S.g.NC);
    }
    ctx->stream_R = S.g.R;
    ctx->stream_Wb = S.g.Wb;
    const StreamGeo& g = S.g;
    cudaStream_t s = ctx->stream;
    struct Cleanup {
        Streamer& S;
        cudaStream_t sc;
        ~Cleanup() {
            cudaStreamSynchronize(sc);
            cudaStreamSynchronize(S.s);
            S.vm.destroy();
            if (S.hkeys) cudaFreeHost(S.hkeys);
            if (S.s) { cudaStreamSynchronize(S.s); if (S.own_s) cudaStreamDestroy(S.s); }
            Buf* bs[] = {&S.tslice, &S.mu, &S.nrm, &S.flat, &S.maxbits, &S.dPw, &S.dIw, &S.sq.scale, &S.sr.scale};
            for (Buf* b : bs) release(*b);
        }
    } cleanup{S, s};

    // window scratch: the largest precompute window is a column window (R + Wb + 1 positions)
    S.wmax = g.R + g.Wb + 4;
    const int64_t wmax = S.wmax;
    MP_CUDA(ctx, ensure(S.tslice, (size_t)d * (wmax + m + 4) * 8));
    MP_CUDA(ctx, ensure(S.mu, (size_t)d * (wmax + 4) * g.tbs));
    MP_CUDA(ctx, ensure(S.nrm, (size_t)d * (wmax + 4) * g.tbs));
    if (g.half) MP_CUDA(ctx, ensure(S.flat, (size_t)d * (wmax + 4) * 3 * 2));
    MP_CUDA(ctx, ensure(S.maxbits, (size_t)d * 2 * sizeof(unsigned long long)));
    MP_CUDA(ctx, ensure(S.dPw, (size_t)d * g.R * 8));
    MP_CUDA(ctx, ensure(S.dIw, (size_t)d * g.R * 8));
    MP_CUDA(ctx, ensure(ctx->flag, sizeof(int)));
    MP_CUDA(ctx, cudaMemsetAsync(ctx->flag.p, 0, sizeof(int), S.s));   // the prep stream runs the checks

    // The caller's T, P and I stay pageable: page-locking them for the call (cudaHostRegister)
    // made the stream tests fail intermittently with launch failures (numpy arrays sharing pages),
    // so the T slices and the output rows are copied from / to pageable memory.
    // virtual arrays at full size (absolute-position layout of run_partial)
    Side* sides[2] = {&S.sq, &S.sr};
    S.sq.T = T;
    S.sr.T = Tr;
    for (int si = 0; si < (self ? 1 : 2); ++si) {
        Side& sd = *sides[si];
        sd.st.name = "st"; sd.stp.name = "stp"; sd.tw.name = "tw"; sd.mup.name = "mup";
        MP_CU(ctx, S.vm.reserve_arr(sd.st, (size_t)n * d * g.sb));
        if (g.half) MP_CU(ctx, S.vm.reserve_arr(sd.stp, (size_t)(n + 1) * d * 16));
        MP_CU(ctx, S.vm.reserve_arr(sd.tw, (size_t)L * g.Dp * g.tb));
        MP_CU(ctx, S.vm.reserve_arr(sd.mup, (size_t)n * g.Dp * g.tb));
        if ((st = S.check_pass(sd)) != MP_OK) return st;
        if (g.half) {
            MP_CUDA(ctx, ensure(sd.scale, (size_t)d * sizeof(double)));
            if ((st = S.half_scale(sd)) != MP_OK) return st;
        }
    }
    S.sq.keys.name = "keys";
    MP_CU(ctx, S.vm.reserve_arr(S.sq.keys, (size_t)n * d * g.kb + 16));
    MP_CUDA(ctx, cudaHostAlloc((void**)&S.hkeys, S.sq.keys.bytes, cudaHostAllocDefault));

    mpk::MainParams mp{};
    mp.st_q = S.sq.st.ptr();
    const Side& rs = self ? S.sq : S.sr;
    mp.st_r = g.half ? rs.stp.ptr() : rs.st.ptr();
    mp.tw_q = S.sq.tw.ptr();
    mp.tw_r = rs.tw.ptr();
    mp.mu_q = S.sq.mup.ptr();
    mp.mu_r = rs.mup.ptr();
    mp.keys = S.sq.keys.ptr();
    mp.n = n; mp.d = (int)d; mp.m = (int)m; mp.H = (int)H;

    ctx->last_launches = 0;
    ctx->last_ms = 0.0;

    // the step list: (row chunk, diagonal band) pairs with cells, in row-chunk order
    struct Step { int64_t B0, B1, q0, q1, i0, i1; Ivl rows, cols; bool last; };
    std::vector<Step> steps;
    std::vector<std::pair<int64_t, int64_t>> empty_chunks;   // row chunks no band reaches
    const int64_t HT = g.HT, NC = g.NC, nq = std::max<int64_t>(1, (n + HT - 1) / HT), qs = g.R / HT;
    const int64_t BW = g.Wb / NC;   // blocks per band
    for (int64_t q0 = 0; q0 < nq; q0 += qs) {
        const int64_t q1 = std::min(nq, q0 + qs), i0 = q0 * HT, i1 = std::min(n, q1 * HT);
        const size_t first = steps.size();
        for (int64_t B0 = 0; B0 < pl.nb; B0 += BW) {
            const int64_t B1 = std::min(pl.nb, B0 + BW);
            const int64_t dlo = pl.dlo + B0 * NC, dhi = std::min(pl.dlo + B1 * NC - 1, pl.dhi);
            const int64_t ra = std::max(i0, -dhi), rb = std::min(i1, n - dlo);   // rows with cells
            if (ra >= rb) continue;
            // windows with a margin of kWinPad positions: the kernels stage one batch of positions
            // past a tile's last row / column (never used by a cell, but read)
            steps.push_back({B0, B1, q0, q1, i0, i1, {i0, std::min<int64_t>(n, i1 + kWinPad)},
                             {std::max<int64_t>(0, ra + dlo - kWinPad), std::min<int64_t>(n, rb + dhi + kWinPad)}, false});
        }
        if (steps.size() == first) empty_chunks.push_back({i0, i1});
        else steps.back().last = true;
    }

    // the tile tables of every step fit the device table buffer allocated here: re-allocating it
    // inside the pipeline would free memory a running kernel reads
    MP_CUDA(ctx, ensure(ctx->seg, (size_t)(2 * nq + 1 + BW + 1) * sizeof(long long)));
    MP_CUDA(ctx, ensure(ctx->counter, sizeof(unsigned long long)));



    // Pipeline: while the fused kernel of step k runs on the compute stream, the host remaps the
    // windows of step k + 1 and the prep stream restores keys and precomputes the new positions.
    // Resident at any time: the windows of two consecutive steps.  Granules outside both are
    // unmapped only after the kernel (and chunk finalize) two steps back has completed.
    cudaStream_t sc = s;            // compute stream (kernels, finalize, output copies)
    cudaStream_t sp = S.s;          // prep stream (remap copies, precompute)
    std::vector<cudaEvent_t> evs;   // per launch: start, end (timing)
    std::vector<cudaEvent_t> done;  // per step: compute stream done through the step (finalize incl.)
    cudaEvent_t prep_ev = nullptr;
    struct EvFree {
        std::vector<cudaEvent_t>& a; std::vector<cudaEvent_t>& b; cudaEvent_t& c;
        ~EvFree() { for (auto e : a) cudaEventDestroy(e); for (auto e : b) cudaEventDestroy(e); if (c) cudaEventDestroy(c); }
    } evfree{evs, done, prep_ev};
    MP_CUDA(ctx, cudaEventCreateWithFlags(&prep_ev, cudaEventDisableTiming));
    Buf tab_pin[3];
    struct PinFree { Buf* b; ~PinFree() { for (int i = 0; i < 3; ++i) if (b[i].p) cudaFreeHost(b[i].p); } } pinfree{tab_pin};
    auto finalize_rows = [&](int64_t i0, int64_t i1) -> mp_status {
        const int64_t w = i1 - i0;
        const double tf0 = Streamer::now();
        MP_CUDA(ctx, mpk::launch_finalize_window(prec, S.sq.keys.ptr(), i0, i1, (int)d, (double*)S.dPw.p,
                                                 (long long*)S.dIw.p, sc));
        MP_CUDA(ctx, cudaMemcpy2DAsync(P + i0, n * 8, S.dPw.p, w * 8, w * 8, d, cudaMemcpyDeviceToHost, sc));
        MP_CUDA(ctx, cudaMemcpy2DAsync(I + i0, n * 8, S.dIw.p, w * 8, w * 8, d, cudaMemcpyDeviceToHost, sc));
        S.t_fin += Streamer::now() - tf0;
        return MP_OK;
    };
    // the window intervals of a step: (series positions of the query side, of the reference side,
    // keys)
    auto windows = [&](const Step& t, std::vector<Ivl>& q, std::vector<Ivl>& r, std::vector<Ivl>& k) {
        if (self) { q.push_back(t.rows); q.push_back(t.cols); k.push_back(t.rows); k.push_back(t.cols); }
        else { q.push_back(t.rows); k.push_back(t.rows); r.push_back(t.cols); }
    };
    size_t ei = 0;   // next empty chunk
    for (size_t k = 0; k < steps.size(); ++k) {
        const Step& t = steps[k];
        // empty row chunks before this step: finalize them synchronously (keys initialised)
        while (ei < empty_chunks.size() && empty_chunks[ei].first < t.i0) {
            MP_CUDA(ctx, cudaStreamSynchronize(sc));
            std::vector<Ivl> kv{{empty_chunks[ei].first, empty_chunks[ei].second}};
            if (k > 0) { std::vector<Ivl> q, r; windows(steps[k - 1], q, r, kv); }
            if ((st = S.remap(S.sq.keys, S.need_mask(S.sq.keys, merge_ivls(kv), (double)d * g.kb, 0), true, t.i0)) != MP_OK)
                return st;
            MP_CUDA(ctx, cudaStreamSynchronize(sp));
            if ((st = finalize_rows(empty_chunks[ei].first, empty_chunks[ei].second)) != MP_OK) return st;
            ++ei;
        }
        // The remap of step k overlaps the kernel of step k - 1 (the windows of both steps stay
        // resident); MP_STREAM_SERIAL=1 waits for that kernel first (no overlap)
        static const bool pipelined = std::getenv("MP_STREAM_SERIAL") == nullptr;
        if (!pipelined && k >= 1) {
            const double t0 = Streamer::now();
            MP_CUDA(ctx, cudaEventSynchronize(done[k - 1]));
            S.t_sync += Streamer::now() - t0;
        }
        if (k >= 2) {
            const double t0 = Streamer::now();
            MP_CUDA(ctx, cudaEventSynchronize(done[k - 2]));
            S.t_sync += Streamer::now() - t0;
        }
        std::vector<Ivl> q, r, kv;
        windows(t, q, r, kv);
        if (k > 0) windows(steps[k - 1], q, r, kv);   // still in use by the running kernel
        // keys of rows below the oldest resident chunk are final: dropped, not saved
        const int64_t final_upto = k > 0 ? steps[k - 1].i0 : t.i0;
        if ((st = S.ensure_side(S.sq, q, &kv, final_upto)) != MP_OK) return st;
        if (!self && (st = S.ensure_side(S.sr, r, nullptr, 0)) != MP_OK) return st;
        MP_CUDA(ctx, cudaEventRecord(prep_ev, sp));
        MP_CUDA(ctx, cudaStreamWaitEvent(sc, prep_ev, 0));
        cudaEvent_t e0, e1, dn;
        MP_CUDA(ctx, cudaEventCreate(&e0));
        evs.push_back(e0);
        MP_CUDA(ctx, cudaEventCreate(&e1));
        evs.push_back(e1);
        MP_CUDA(ctx, cudaEventRecord(e0, sc));
        if ((st = enqueue_tiles(ctx, sc, kernel_prec(prec, m, mpk::pick_variant(prec, (int)d)), self, mp, pl, t.B0, t.B1,
                                t.q0, t.q1, false, &tab_pin[k % 3])) != MP_OK)
            return st;
        MP_CUDA(ctx, cudaEventRecord(e1, sc));
        // rows [i0, i1) are final after the chunk's last band: later chunks only touch rows >= i1
        // and (self-join) columns > their rows; rows no band reached keep the empty key (G3)
        if (t.last && (st = finalize_rows(t.i0, t.i1)) != MP_OK) return st;
        MP_CUDA(ctx, cudaEventCreateWithFlags(&dn, cudaEventDisableTiming));
        done.push_back(dn);
        MP_CUDA(ctx, cudaEventRecord(dn, sc));
    }
    while (ei < empty_chunks.size()) {   // trailing row chunks no band reaches
        MP_CUDA(ctx, cudaStreamSynchronize(sc));
        std::vector<Ivl> kv{{empty_chunks[ei].first, empty_chunks[ei].second}};
        if ((st = S.remap(S.sq.keys, S.need_mask(S.sq.keys, kv, (double)d * g.kb, 0), true, empty_chunks[ei].first)) != MP_OK)
            return st;
        MP_CUDA(ctx, cudaStreamSynchronize(sp));
        if ((st = finalize_rows(empty_chunks[ei].first, empty_chunks[ei].second)) != MP_OK) return st;
        ++ei;
    }
    if (std::getenv("MP_STREAM_PROFILE"))
        std::fprintf(stderr, "mp_compute_stream: host s sync %.3f remap %.3f (key saves %.3f unmap %.3f map+restore %.3f) "
                     "precompute %.3f finalize %.3f\n", S.t_sync, S.t_remap, S.t_save, S.t_unmap, S.t_map, S.t_pre, S.t_fin);
    MP_CUDA(ctx, cudaStreamSynchronize(s));
    double tot = 0;
    for (size_t k = 0; k + 1 < evs.size(); k += 2) {
        float ms = 0.f;
        MP_CUDA(ctx, cudaEventElapsedTime(&ms, evs[k], evs[k + 1]));
        tot += ms;
    }
    ctx->last_ms = tot;
    ctx->stream_timed = true;
    ctx->stream_peak = (int64_t)S.vm.peak;
    ctx->stream_launches = ctx->last_launches;
    return finish_partial(ctx, s);
}

}  // namespace

extern "C" {

const char* mp_version(void) { return "mstamp-b200 0.1 (sm_100a)"; }

mp_status mp_init(mp_ctx** out, const mp_config* cfg) {
    if (!out) return MP_ERR_INVALID;
    *out = nullptr;
    mp_ctx* ctx = new (std::nothrow) mp_ctx();
    if (!ctx) return MP_ERR_NOMEM;
    if (cfg) {
        ctx->device = cfg->device;
        for (int i = 0; i < 4; ++i) ctx->H[i] = cfg->reseed_h[i];
        ctx->H[4] = cfg->reseed_h[2];  // FP16C follows FP16
        ctx->H[5] = cfg->reseed_h[3];  // FP16CK follows MIXED
        if (cfg->seed_mode != MP_SEEDS_DIRECT && cfg->seed_mode != MP_SEEDS_TC) { delete ctx; return MP_ERR_INVALID; }
        ctx->seed_mode = cfg->seed_mode;
    }
    for (int i = 0; i < 6; ++i)
        if (ctx->H[i] < 0 || ctx->H[i] > (int64_t(1) << 30)) { delete ctx; return MP_ERR_INVALID; }
    int ndev = 0;
    cudaError_t e = cudaGetDeviceCount(&ndev);
    if (e != cudaSuccess || ndev == 0) { delete ctx; return MP_ERR_CUDA; }
    if (ctx->device < 0 || ctx->device >= ndev) { delete ctx; return MP_ERR_INVALID; }
    if (cudaSetDevice(ctx->device) != cudaSuccess) { delete ctx; return MP_ERR_CUDA; }
    cudaDeviceGetAttribute(&ctx->nsm, cudaDevAttrMultiProcessorCount, ctx->device);
    if (cudaStreamCreateWithFlags(&ctx->stream, cudaStreamNonBlocking) != cudaSuccess ||
        cudaEventCreate(&ctx->ev0) != cudaSuccess || cudaEventCreate(&ctx->ev1) != cudaSuccess) {
        mp_free(ctx);
        return MP_ERR_CUDA;
    }
    *out = ctx;
    return MP_OK;
}

void mp_free(mp_ctx* ctx) {
    if (!ctx) return;
    cudaSetDevice(ctx->device);
    Buf* bufs[] = {&ctx->dT, &ctx->dTr, &ctx->st_q, &ctx->st_r, &ctx->tw_q, &ctx->tw_r, &ctx->mu_q,
                   &ctx->mu_r, &ctx->mup_q, &ctx->mup_r, &ctx->nrm, &ctx->keys, &ctx->ext, &ctx->seg, &ctx->counter, &ctx->dP,
                   &ctx->dI, &ctx->flag, &ctx->stp_q, &ctx->stp_r, &ctx->scale, &ctx->scale_r, &ctx->maxbits, &ctx->flat,
                   &ctx->seedtab};
    for (Buf* b : bufs) release(*b);
    if (ctx->hflag) cudaFreeHost(ctx->hflag);
    if (ctx->ev0) cudaEventDestroy(ctx->ev0);
    if (ctx->ev1) cudaEventDestroy(ctx->ev1);
    if (ctx->stream) cudaStreamDestroy(ctx->stream);
    delete ctx;
}

const char* mp_last_error(const mp_ctx* ctx) {
    if (!ctx) return "no context";
    return ctx->err.c_str();
}

int64_t mp_key_words(int64_t d, int64_t n, mp_precision prec) {
    return d * n * (prec == MP_FP64 ? 2 : 1);
}

mp_status mp_plan_bands(int64_t d, int64_t n, int64_t m, mp_precision prec, int64_t exclusion,
                        int self_join, int world, int64_t* block_begin, int64_t* cells) {
    if (world < 1 || !block_begin || !cells || d < 1 || n < 2 || m < 2 || prec < 0 || prec > 5)
        return MP_ERR_INVALID;
    if (self_join && exclusion < 0) exclusion = (m + 3) / 4;
    Plan pl = build_plan(d, n, exclusion, self_join != 0, prec, default_h(prec, m));
    if (pl.nb == 0) {
        for (int g = 0; g <= world; ++g) block_begin[g] = 0;
        for (int g = 0; g < world; ++g) cells[g] = 0;
        return MP_OK;
    }
    std::vector<int64_t> bb = band_blocks(pl, world);
    for (int g = 0; g <= world; ++g) block_begin[g] = bb[g];
    for (int g = 0; g < world; ++g) cells[g] = (int64_t)(pl.cells[bb[g + 1]] - pl.cells[bb[g]]);
    return MP_OK;
}

mp_status mp_plan_diagonals(int64_t d, int64_t n, int64_t m, mp_precision prec, int64_t exclusion,
                            int self_join, int world, int64_t* diag_begin) {
    if (world < 1 || !diag_begin || d < 1 || n < 2 || m < 2 || prec < 0 || prec > 5) return MP_ERR_INVALID;
    if (self_join && exclusion < 0) exclusion = (m + 3) / 4;
    Plan pl = build_plan(d, n, exclusion, self_join != 0, prec, default_h(prec, m));
    if (pl.nb == 0) {
        for (int g = 0; g <= world; ++g) diag_begin[g] = pl.dlo;
        return MP_OK;
    }
    std::vector<int64_t> bb = band_blocks(pl, world);
    for (int g = 0; g <= world; ++g) diag_begin[g] = std::min<int64_t>(pl.dlo + bb[g] * pl.nc, pl.dhi + 1);
    return MP_OK;
}

mp_status mp_partial_device(mp_ctx* ctx, void* cuda_stream, const double* dT, const double* dTr,
                            int64_t d, int64_t n, int64_t m, mp_precision prec, int64_t exclusion,
                            int rank, int world, int64_t* dKeys) {
    if (!ctx) return MP_ERR_INVALID;
    mp_status st = validate(ctx, dT, d, n, m, prec);
    if (st != MP_OK) return st;
    if (!dKeys || world < 1 || rank < 0 || rank >= world) return fail(ctx, MP_ERR_INVALID, "bad rank/world/keys");
    MP_CUDA(ctx, cudaSetDevice(ctx->device));
    cudaStream_t s = (cudaStream_t)cuda_stream;  // NULL = the legacy default stream
    st = run_partial(ctx, s, dT, dTr, d, n, m, prec, exclusion, rank, world);
    if (st != MP_OK) return st;
    MP_CUDA(ctx, mpk::launch_keys_to_ext(prec, ctx->keys.p, dKeys, n * d, s));
    return finish_partial(ctx, s);
}

mp_status mp_key_mask_device(mp_ctx* ctx, void* cuda_stream, int64_t d, int64_t n, int64_t* dKeys,
                             const int64_t* dGlobalV) {
    if (!ctx || !dKeys || !dGlobalV || d < 1 || n < 1) return fail(ctx, MP_ERR_INVALID, "bad arguments");
    MP_CUDA(ctx, cudaSetDevice(ctx->device));
    cudaStream_t s = (cudaStream_t)cuda_stream;  // NULL = the legacy default stream
    MP_CUDA(ctx, mpk::launch_key_mask(n * d, (long long*)dKeys, (const long long*)dGlobalV, s));
    return MP_OK;
}

mp_status mp_finalize_device(mp_ctx* ctx, void* cuda_stream, int64_t d, int64_t n, mp_precision prec,
                             const int64_t* dKeys, double* dP, int64_t* dI) {
    if (!ctx || !dKeys || !dP || !dI || d < 1 || n < 1) return fail(ctx, MP_ERR_INVALID, "bad arguments");
    MP_CUDA(ctx, cudaSetDevice(ctx->device));
    cudaStream_t s = (cudaStream_t)cuda_stream;  // NULL = the legacy default stream
    MP_CUDA(ctx, mpk::launch_finalize(prec, dKeys, n, (int)d, dP, (long long*)dI, s));
    return MP_OK;
}

mp_status mp_compute_device(mp_ctx* ctx, void* cuda_stream, const double* dT, const double* dTr,
                            int64_t d, int64_t n, int64_t m, mp_precision prec, int64_t exclusion,
                            double* dP, int64_t* dI) {
    if (!ctx) return MP_ERR_INVALID;
    mp_status st = validate(ctx, dT, d, n, m, prec);
    if (st != MP_OK) return st;
    if (!dP || !dI) return fail(ctx, MP_ERR_INVALID, "P or I is NULL");
    MP_CUDA(ctx, cudaSetDevice(ctx->device));
    cudaStream_t s = (cudaStream_t)cuda_stream;  // NULL = the legacy default stream
    st = run_partial(ctx, s, dT, dTr, d, n, m, prec, exclusion, 0, 1);
    if (st != MP_OK) return st;
    if (prec == MP_FP64) {
        MP_CUDA(ctx, ensure(ctx->ext, (size_t)n * d * 16));
        MP_CUDA(ctx, mpk::launch_keys_to_ext(prec, ctx->keys.p, ctx->ext.p, n * d, s));
        MP_CUDA(ctx, mpk::launch_finalize(prec, ctx->ext.p, n, (int)d, dP, (long long*)dI, s));
    } else {
        MP_CUDA(ctx, mpk::launch_finalize(prec, ctx->keys.p, n, (int)d, dP, (long long*)dI, s));
    }
    return finish_partial(ctx, s);
}

mp_status mp_compute(mp_ctx* ctx, const double* T, const double* Tr, int64_t d, int64_t n, int64_t m,
                     mp_precision prec, int64_t exclusion, double* P, int64_t* I) {
    if (!ctx) return MP_ERR_INVALID;
    mp_status st = validate(ctx, T, d, n, m, prec);
    if (st != MP_OK) return st;
    if (!P || !I) return fail(ctx, MP_ERR_INVALID, "P or I is NULL");
    const int64_t L = n + m - 1;  // non-finite input is rejected by the device check in run_partial
    MP_CUDA(ctx, cudaSetDevice(ctx->device));
    cudaStream_t s = ctx->stream;
    MP_CUDA(ctx, ensure(ctx->dT, (size_t)d * L * 8));
    MP_CUDA(ctx, cudaMemcpyAsync(ctx->dT.p, T, (size_t)d * L * 8, cudaMemcpyHostToDevice, s));
    if (Tr) {
        MP_CUDA(ctx, ensure(ctx->dTr, (size_t)d * L * 8));
        MP_CUDA(ctx, cudaMemcpyAsync(ctx->dTr.p, Tr, (size_t)d * L * 8, cudaMemcpyHostToDevice, s));
    }
    MP_CUDA(ctx, ensure(ctx->dP, (size_t)d * n * 8));
    MP_CUDA(ctx, ensure(ctx->dI, (size_t)d * n * 8));
    st = mp_compute_device(ctx, s, (const double*)ctx->dT.p, Tr ? (const double*)ctx->dTr.p : nullptr, d, n,
                           m, prec, exclusion, (double*)ctx->dP.p, (int64_t*)ctx->dI.p);
    if (st != MP_OK) return st;
    MP_CUDA(ctx, cudaMemcpyAsync(P, ctx->dP.p, (size_t)d * n * 8, cudaMemcpyDeviceToHost, s));
    MP_CUDA(ctx, cudaMemcpyAsync(I, ctx->dI.p, (size_t)d * n * 8, cudaMemcpyDeviceToHost, s));
    MP_CUDA(ctx, cudaStreamSynchronize(s));
    return MP_OK;
}

mp_status mp_selftest_sort_scan(mp_ctx* ctx, int64_t d, int64_t count, const float* in, float* out) {
    if (!ctx || !in || !out || d < 1 || d > MP_MAX_D || count < 1) return fail(ctx, MP_ERR_INVALID, "bad arguments");
    MP_CUDA(ctx, cudaSetDevice(ctx->device));
    cudaStream_t s = ctx->stream;
    Buf a, b;
    const size_t bytes = (size_t)count * d * sizeof(float);
    MP_CUDA(ctx, ensure(a, bytes));
    cudaError_t e = ensure(b, bytes);
    if (e == cudaSuccess) e = cudaMemcpyAsync(a.p, in, bytes, cudaMemcpyHostToDevice, s);
    if (e == cudaSuccess) e = mpk::launch_selftest_sort_scan((int)d, count, (const float*)a.p, (float*)b.p, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(out, b.p, bytes, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    release(a);
    release(b);
    return e == cudaSuccess ? MP_OK : cuda_fail(ctx, e, "mp_selftest_sort_scan");
}

mp_status mp_selftest_seeds(mp_ctx* ctx, const double* T, const double* Tr, int64_t d, int64_t n, int64_t m,
                            mp_precision prec, int64_t H, int64_t r_lo, int64_t r_hi, double* out,
                            double* scale_out) {
    if (!ctx) return MP_ERR_INVALID;
    mp_status st = validate(ctx, T, d, n, m, prec);
    if (st != MP_OK) return st;
    if (!out || !scale_out || (prec != MP_MIXED && prec != MP_FP16CK) || H < 1 || r_lo < 0 || r_hi <= r_lo ||
        r_hi > (n + H - 1) / H)
        return fail(ctx, MP_ERR_INVALID, "bad arguments");
    MP_CUDA(ctx, cudaSetDevice(ctx->device));
    cudaStream_t s = ctx->stream;
    const int64_t L = n + m - 1;
    MP_CUDA(ctx, ensure(ctx->dT, (size_t)d * L * 8));
    MP_CUDA(ctx, cudaMemcpyAsync(ctx->dT.p, T, (size_t)d * L * 8, cudaMemcpyHostToDevice, s));
    if (Tr) {
        MP_CUDA(ctx, ensure(ctx->dTr, (size_t)d * L * 8));
        MP_CUDA(ctx, cudaMemcpyAsync(ctx->dTr.p, Tr, (size_t)d * L * 8, cudaMemcpyHostToDevice, s));
    }
    const double* dT = (const double*)ctx->dT.p;
    const double* dTr = Tr ? (const double*)ctx->dTr.p : nullptr;
    st = run_partial(ctx, s, dT, dTr, d, n, m, prec, 0, 0, 1, true);
    if (st != MP_OK) return st;
    const bool self = Tr == nullptr;
    mpk::SeedParams sp{};
    sp.Tq = dT; sp.Tr = self ? dT : dTr;
    sp.scale_q = (const double*)ctx->scale.p;
    sp.scale_r = (const double*)(self ? ctx->scale.p : ctx->scale_r.p);
    sp.mu_q = (const float*)ctx->mu_q.p;
    sp.mu_r = (const float*)(self ? ctx->mu_q.p : ctx->mu_r.p);
    sp.n = n; sp.d = (int)d; sp.m = (int)m; sp.H = (int)H;
    sp.r_lo = r_lo; sp.r_hi = r_hi; sp.j_lo = 0; sp.j_hi = n; sp.ldj = (n + 7) / 8 * 8;
    const size_t cnt = (size_t)(r_hi - r_lo) * d * sp.ldj;
    Buf tb;
    MP_CUDA(ctx, ensure(tb, cnt * 2));
    sp.tab = tb.p;
    std::vector<__half> h(cnt);
    cudaError_t e = mpk::launch_seed_gemm(sp, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(h.data(), tb.p, cnt * 2, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(scale_out, ctx->scale.p, d * 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess && !self) e = cudaMemcpyAsync(scale_out + d, ctx->scale_r.p, d * 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    release(tb);
    if (e != cudaSuccess) return cuda_fail(ctx, e, "mp_selftest_seeds");
    for (int64_t r = 0; r < r_hi - r_lo; ++r)       // unpack [r][dim][ldj] half -> [r][dim][n] double
        for (int64_t k = 0; k < d; ++k)
            for (int64_t j = 0; j < n; ++j)
                out[(r * d + k) * n + j] = (double)__half2float(h[(r * d + k) * sp.ldj + j]);
    return finish_partial(ctx, s);
}

mp_status mp_selftest_precompute(mp_ctx* ctx, const double* T, int64_t d, int64_t n, int64_t m,
                                 mp_precision prec, double* df, double* dg, double* a) {
    if (!ctx) return MP_ERR_INVALID;
    mp_status st = validate(ctx, T, d, n, m, prec);
    if (st != MP_OK) return st;
    if (!df || !dg || !a || (prec != MP_FP64 && prec != MP_FP32)) return fail(ctx, MP_ERR_INVALID, "bad arguments");
    MP_CUDA(ctx, cudaSetDevice(ctx->device));
    cudaStream_t s = ctx->stream;
    const int64_t L = n + m - 1;
    MP_CUDA(ctx, ensure(ctx->dT, (size_t)d * L * 8));
    MP_CUDA(ctx, cudaMemcpyAsync(ctx->dT.p, T, (size_t)d * L * 8, cudaMemcpyHostToDevice, s));
    const mpk::Variant var = mpk::pick_variant(prec, (int)d);
    mpk::PreParams pp{};
    pp.n = n; pp.d = (int)d; pp.m = (int)m; pp.Dp = var.DL * var.G;
    full_window(pp, n, L);
    if (var.ctab) { pp.pm_G = var.G; pp.pm_DL = var.DL; }
    const size_t eb = elt_bytes(prec), tbs = 8;
    MP_CUDA(ctx, ensure(ctx->nrm, (size_t)n * d * tbs));
    pp.nrm32 = (float*)ctx->nrm.p; pp.nrm64 = (double*)ctx->nrm.p;
    MP_CUDA(ctx, ensure(ctx->st_q, (size_t)n * d * 4 * eb));
    MP_CUDA(ctx, ensure(ctx->mu_q, (size_t)n * d * tbs));
    MP_CUDA(ctx, ensure(ctx->mup_q, (size_t)n * pp.Dp * eb));
    MP_CUDA(ctx, ensure(ctx->tw_q, (size_t)L * pp.Dp * eb));
    pp.T = (const double*)ctx->dT.p; pp.st = ctx->st_q.p; pp.mu = ctx->mu_q.p; pp.mup = ctx->mup_q.p; pp.tw = ctx->tw_q.p;
    MP_CUDA(ctx, mpk::launch_precompute(prec, pp, s));
    Buf o;
    MP_CUDA(ctx, ensure(o, (size_t)n * d * 3 * 8));
    double* od = (double*)o.p;
    cudaError_t e = mpk::launch_selftest_unpack(prec, ctx->st_q.p, n, (int)d, od, od + n * d, od + 2 * n * d, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(df, od, (size_t)n * d * 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(dg, od + n * d, (size_t)n * d * 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaMemcpyAsync(a, od + 2 * n * d, (size_t)n * d * 8, cudaMemcpyDeviceToHost, s);
    if (e == cudaSuccess) e = cudaStreamSynchronize(s);
    release(o);
    return e == cudaSuccess ? MP_OK : cuda_fail(ctx, e, "mp_selftest_precompute");
}

mp_status mp_last_timing(const mp_ctx* ctx, double* main_kernel_ms, int64_t* launches) {
    if (!ctx || !main_kernel_ms || !launches) return MP_ERR_INVALID;
    *launches = ctx->last_launches;
    *main_kernel_ms = 0.0;
    if (ctx->stream_timed) {   // mp_compute_stream: the sum over its launches (measured there)
        *main_kernel_ms = ctx->last_ms;
        return MP_OK;
    }
    if (ctx->last_launches > 0) {
        float ms = 0.f;
        if (cudaEventSynchronize(ctx->ev1) != cudaSuccess) return MP_ERR_CUDA;
        if (cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1) != cudaSuccess) return MP_ERR_CUDA;
        *main_kernel_ms = ms;
    }
    return MP_OK;
}

mp_status mp_plan_stream(int64_t d, int64_t n, int64_t m, mp_precision prec, int64_t exclusion, int self_join,
                         int64_t device_bytes, int64_t granularity, int64_t* rows_per_chunk,
                         int64_t* diagonals_per_band) {
    if (!rows_per_chunk || !diagonals_per_band || d < 1 || d > MP_MAX_D || n < 2 || m < 2 || prec < 0 ||
        prec > 5 || granularity < 1 || device_bytes < 1)
        return MP_ERR_INVALID;
    if (self_join && exclusion < 0) exclusion = (m + 3) / 4;
    const Plan pl = build_plan(d, n, exclusion, self_join != 0, prec, default_h(prec, m));
    StreamGeo g;
    mp_status st = plan_stream(nullptr, d, n, m, prec, exclusion, self_join != 0, device_bytes, (size_t)granularity, pl, g);
    if (st != MP_OK) return st;
    *rows_per_chunk = g.R;
    *diagonals_per_band = g.Wb;
    return MP_OK;
}

mp_status mp_compute_stream(mp_ctx* ctx, const double* T, const double* Tr, int64_t d, int64_t n, int64_t m,
                            mp_precision prec, int64_t exclusion, int64_t device_bytes, double* P, int64_t* I) {
    if (!ctx) return MP_ERR_INVALID;
    mp_status st = validate(ctx, T, d, n, m, prec);
    if (st != MP_OK) return st;
    if (!P || !I) return fail(ctx, MP_ERR_INVALID, "P or I is NULL");
    if (device_bytes < 1) return fail(ctx, MP_ERR_INVALID, "device_bytes must be positive");
    MP_CUDA(ctx, cudaSetDevice(ctx->device));
    return run_stream(ctx, T, Tr, d, n, m, prec, exclusion, device_bytes, P, I);
}

mp_status mp_last_stream_info(const mp_ctx* ctx, int64_t* rows_per_chunk, int64_t* diagonals_per_band,
                              int64_t* peak_device_bytes, int64_t* launches) {
    if (!ctx || !rows_per_chunk || !diagonals_per_band || !peak_device_bytes || !launches) return MP_ERR_INVALID;
    *rows_per_chunk = ctx->stream_R;
    *diagonals_per_band = ctx->stream_Wb;
    *peak_device_bytes = ctx->stream_peak;
    *launches = ctx->stream_launches;
    return MP_OK;
}

}  // extern "C"

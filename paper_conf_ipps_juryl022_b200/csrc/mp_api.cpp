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

#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstdio>
#include <cstring>
#include <string>
#include <vector>

namespace {

constexpr int64_t kDefaultH[5] = {4096, 1024, 256, 256, 256};  // FP64, FP32, FP16, MIXED, FP16C (upper bounds)

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
    int64_t H[5] = {0, 0, 0, 0, 0};
    std::string err;
    // cached scratch
    Buf dT, dTr, st_q, st_r, tw_q, tw_r, mu_q, mu_r, mup_q, mup_r, nrm, keys, ext, seg, counter, dP, dI, flag;
    Buf stp_q, stp_r, scale, maxbits, flat;  // FP16 / Mixed precompute
    cudaEvent_t ev0 = nullptr, ev1 = nullptr;
    int* hflag = nullptr;   // pinned read-back of the non-finite flag
    double last_ms = 0.0;
    int64_t last_launches = 0;
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
    if (prec < 0 || prec > 4) return fail(ctx, MP_ERR_INVALID, "unknown precision");
    if (prec == MP_FP64 && d > 512) return fail(ctx, MP_ERR_UNSUPPORTED, "FP64 supports d <= 512");
    return MP_OK;
}

// Device pipeline: keys for band (rank, world) of the tile plan, internal key format.
mp_status run_partial(mp_ctx* ctx, cudaStream_t s, const double* dT, const double* dTr, int64_t d,
                      int64_t n, int64_t m, int prec, int64_t excl, int rank, int world) {
    const bool self = dTr == nullptr;
    const int64_t L = n + m - 1;
    const size_t eb = elt_bytes(prec);
    // re-seeds happen at staging-batch starts (every kernel steps in batches of 1, 2 or 4 rows),
    // so the interval is rounded up to a multiple of 8: then every re-seed row i = 0 mod H is a
    // batch start in every kernel variant (include/mp.h, mp_config.reseed_h)
    int64_t H = ctx->H[prec] > 0 ? ctx->H[prec] : default_h(prec, m);
    H = std::min<int64_t>((H + 7) / 8 * 8, int64_t(1) << 30);
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
    const bool half = prec == MP_FP16 || prec == MP_MIXED || prec == MP_FP16C;
    const size_t sb = half ? 16 : 4 * eb;                                   // stats entry bytes
    const size_t tb = prec == MP_FP64 ? 8 : ((prec == MP_FP16 || prec == MP_FP16C) ? 2 : 4);  // precalc value bytes
    const size_t tbs = prec == MP_FP32 ? 8 : tb;  // window stats scratch (FP32 mode: FP64 precalc, reading R1')
    const mpk::Variant var = mpk::pick_variant(prec, (int)d);
    const int Dp = var.DL * var.G;
    mpk::PreParams pp{};
    pp.n = n; pp.d = (int)d; pp.m = (int)m; pp.Dp = Dp;
    if (var.ctab) { pp.pm_G = var.G; pp.pm_DL = var.DL; }
    MP_CUDA(ctx, ensure(ctx->nrm, (size_t)n * d * tbs));
    pp.nrm32 = (float*)ctx->nrm.p; pp.nrm64 = (double*)ctx->nrm.p;
    if (half) {
        MP_CUDA(ctx, ensure(ctx->scale, (size_t)d * sizeof(double)));
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
        pp.st = B[0]->p; pp.st_pair = B[1]->p; pp.mu = B[2]->p; pp.mup = B[3]->p; pp.tw = B[4]->p;
        MP_CUDA(ctx, mpk::launch_precompute(prec, pp, s));
    }

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
        const long long t_begin = pl.seg[bb[rank]], t_end = pl.seg[bb[rank + 1]];
        // segment-major tile order over the band's blocks [B0, B1): for row segment q the
        // blocks with a tile in it are contiguous, [first b with qlo_b <= q, first b with
        // qhi_b <= q), because a block's first and last rows never increase with b
        const int64_t B0 = bb[rank], B1 = bb[rank + 1], HT = pl.H;
        const int64_t nq = std::max<int64_t>(1, (n + HT - 1) / HT);
        auto qlo = [&](int64_t b) {
            const int64_t d1 = std::min(pl.dlo + b * pl.nc + pl.nc - 1, pl.dhi);
            return std::max<int64_t>(0, -d1) / HT;
        };
        auto qhi = [&](int64_t b) {
            const int64_t d0 = pl.dlo + b * pl.nc;
            return (std::min<int64_t>(n, n - std::max<int64_t>(d0, 0)) + HT - 1) / HT;
        };
        auto first_b = [&](auto pred) {  // first b in [B0, B1) with pred(b) (monotone), else B1
            int64_t lo = B0, hi = B1;
            while (lo < hi) {
                const int64_t mid = (lo + hi) / 2;
                if (pred(mid)) hi = mid; else lo = mid + 1;
            }
            return lo;
        };
        std::vector<long long> qtab(2 * nq + 1);  // [q_prefix (nq + 1) | q_block0 (nq) | ...]
        qtab[0] = 0;
        for (int64_t q = 0; q < nq; ++q) {
            const int64_t bs = first_b([&](int64_t b) { return qlo(b) <= q; });
            const int64_t be = first_b([&](int64_t b) { return qhi(b) <= q; });
            qtab[q + 1] = qtab[q] + std::max<int64_t>(0, be - bs);
            qtab[nq + 1 + q] = bs;
        }
        if (qtab[nq] != t_end - t_begin) return fail(ctx, MP_ERR_INVALID, "internal: tile plan mismatch");
        qtab.insert(qtab.end(), pl.seg.begin(), pl.seg.end());  // [.. | seg_prefix (nb + 1)]
        MP_CUDA(ctx, ensure(ctx->seg, qtab.size() * sizeof(long long)));
        MP_CUDA(ctx, cudaMemcpyAsync(ctx->seg.p, qtab.data(), qtab.size() * sizeof(long long),
                                     cudaMemcpyHostToDevice, s));
        MP_CUDA(ctx, ensure(ctx->counter, sizeof(unsigned long long)));
        MP_CUDA(ctx, cudaMemsetAsync(ctx->counter.p, 0, sizeof(unsigned long long), s));
        if (t_end > t_begin) {
            mpk::MainParams mp{};
            mp.st_q = ctx->st_q.p;
            mp.st_r = self ? ctx->st_q.p : ctx->st_r.p;
            if (half) mp.st_r = self ? ctx->stp_q.p : ctx->stp_r.p;   // columns: pair format
            mp.tw_q = ctx->tw_q.p;
            mp.tw_r = self ? ctx->tw_q.p : ctx->tw_r.p;
            mp.mu_q = ctx->mup_q.p;
            mp.mu_r = self ? ctx->mup_q.p : ctx->mup_r.p;
            mp.keys = ctx->keys.p;
            mp.order = var.cta ? 0 : 1;   // decode_tile (mp_diag.cuh) says why
            mp.q_prefix = (const long long*)ctx->seg.p;
            mp.q_block0 = (const long long*)ctx->seg.p + nq + 1;
            mp.nq = nq;
            mp.seg_prefix = (const long long*)ctx->seg.p + 2 * nq + 1;
            mp.nb = pl.nb;
            mp.t_begin = t_begin;
            mp.t_count = t_end - t_begin;
            mp.counter = (unsigned long long*)ctx->counter.p;
            mp.n = n; mp.d = (int)d; mp.m = (int)m; mp.H = (int)H; mp.HT = pl.H;
            mp.delta_lo = pl.dlo; mp.delta_hi = pl.dhi;
            const int bps = std::max(1, mpk::main_blocks_per_sm(prec, (int)d, self));
            const long long want_warps = mp.t_count;
            long long grid = (long long)ctx->nsm * bps;
            const int wpb = std::max(1, mpk::variant_warps_per_block(prec, (int)d, self));
            grid = std::min<long long>(grid, (want_warps + wpb - 1) / wpb);
            grid = std::max<long long>(grid, 1);
            MP_CUDA(ctx, cudaEventRecord(ctx->ev0, s));
            MP_CUDA(ctx, mpk::launch_main(prec, self, mp, (int)grid, s));
            MP_CUDA(ctx, cudaEventRecord(ctx->ev1, s));
            ctx->last_launches = 1;
        }
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
    }
    for (int i = 0; i < 5; ++i)
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
                   &ctx->dI, &ctx->flag, &ctx->stp_q, &ctx->stp_r, &ctx->scale, &ctx->maxbits, &ctx->flat};
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
    if (world < 1 || !block_begin || !cells || d < 1 || n < 2 || m < 2 || prec < 0 || prec > 4)
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
    if (world < 1 || !diag_begin || d < 1 || n < 2 || m < 2 || prec < 0 || prec > 4) return MP_ERR_INVALID;
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
    if (ctx->last_launches > 0) {
        float ms = 0.f;
        if (cudaEventSynchronize(ctx->ev1) != cudaSuccess) return MP_ERR_CUDA;
        if (cudaEventElapsedTime(&ms, ctx->ev0, ctx->ev1) != cudaSuccess) return MP_ERR_CUDA;
        *main_kernel_ms = ms;
    }
    return MP_OK;
}

}  // extern "C"

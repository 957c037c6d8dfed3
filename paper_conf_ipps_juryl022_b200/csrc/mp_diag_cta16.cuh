#pragma once
// mp_diag_cta16.cuh -- half-precision (FP16 / Mixed / FP16C) fused diagonal kernel for large d:
// the block-cooperative tiles of mp_diag_cta.cuh with the half2 cell pairs of mp_diag16.cuh.
//
// Method per cell (unchanged): QT recurrence (Eq. 1), distance (Eq. 1,
// L500-507), d-way sort (in-lane Batcher network + warp-shuffle bitonic merge across the G
// lanes of a cell) and inclusive scan (Eq. 2), filtered min / argmin into the row and
// column profile (Eq. 3; self-join symmetry, reading G13).  Arithmetic as in the
// paper's FP16 modes (Fig. 1 table; Sec. III-C): half2, two cells per lane.
//
// Staging (why this kernel exists): at large d a warp-private ring costs d x 24-32 B per
// position and a warp holds only 32/G lane-cells, so few warps fit per SM.  Here the NW warps
// of a block step through one tile together: the block's 2 NT/G cells are consecutive
// diagonals in the SAME row, so per step the block stages one row position (8 B per dim:
// df, dg, a, threshold as halves) and one column pair slot (16 B per dim: the pair (c, c+1) as
// half2, so one LDS.128 feeds both cells of a lane) into rings shared by all its warps.
//
// Profile updates are lane-local and write through: a lane whose prefix sum beats the staged
// half threshold does a global RED.MIN.64 on the merge key ((float bits of the half value) << 32
// | index: lexicographic (value, index) min, reading G2) and lowers the ring's threshold hint
// with a plain 16-bit store.  A hint is always a value that was merged, so it is never below the
// true best (a racing store can only leave it higher: more slow-path visits, never a missed
// update).  No eviction pass, no key ring.  Thresholds enter the ring as the key's FP32 value
// word (cp.async into a float staging slot); after its own copies land each thread converts the
// entries it staged to half (exact: every best is a half value), then one block barrier per
// batch publishes them.
#include "mp_diag16.cuh"

#ifndef MP_CTAH_NW
#define MP_CTAH_NW 4       // 0 switches the block-cooperative half kernel off
#endif
#ifndef MP_CTAH_MIN_DP
#define MP_CTAH_MIN_DP 64  // smallest padded d that takes it
#endif

namespace mpk {


// Per lane-group-size launch shape (measured on one B200, Mixed self-joins of d = 64 / 128 / 256,
// n = 32768 / 16384 / 8192): warps per block and steps per staging batch (one block barrier per
// batch).  d = 64: 4 warps, SB = 2 (61.0 -> 58.9 ms); d = 128: 8 warps (45.7 -> 39.5 ms);
// d = 256: 4 warps, SB = 1 (SB = 2: 31.3 -> 34.9 ms, 8 warps: 33.7 ms).
template <int G> struct CtaShapeH {
    static constexpr int NW = MP_CTAH_NW == 0 ? 0 : (G == 16 ? 8 : 4);
    static constexpr int SB = G == 8 ? 2 : 1;
    static constexpr int MINB = NW == 8 ? 2 : 4;   // 128 registers per thread
};

template <int DL, int G, int NW> struct CtaGeoH {
    static constexpr int NT = 32 * NW;   // threads per block
    static constexpr int NP = NT / G;    // cell pairs per block tile
    static constexpr int NCC = 2 * NP;   // cells (diagonals) per block tile
    static constexpr int D = DL * G;
    static constexpr int SB = CtaShapeH<G>::SB;
    // row slots: current batch + prefetch (+1 batch margin); column pair slots (by first
    // column): the live span [s0 - 1, s0 + SB + NCC - 2], the fixup target s0 + SB + NCC - 1
    // and the prefetch [s0 + SB + NCC, s0 + 2 SB + NCC) never share a slot
    static constexpr int RR = 3 * SB;
    static constexpr int RC = 3 * SB + NCC + 2;
    static constexpr size_t a16(size_t x) { return (x + 15) & ~(size_t)15; }
    static constexpr size_t col_bytes = (size_t)RC * D * sizeof(H4);
    static constexpr size_t row_bytes = a16((size_t)RR * D * sizeof(RH));
    static constexpr size_t stg_bytes = a16((size_t)(RR + RC) * D * sizeof(float));
    static constexpr size_t bytes = col_bytes + row_bytes + stg_bytes + 16 /* tile index */ + 16 /* mbarrier */;
};

#ifndef MP_CTAH_TMA
#define MP_CTAH_TMA 0   // stage each entering position's statistics by one TMA bulk copy (measured:
                        // C3 Mixed 3529 -> 3701 ms, X64 60.1 -> 62.8 ms against cp.async: off)
#endif

// Seeds of a cell pair from the tensor-core seed table (MP_SEEDS_TC, mp_seed_tc.cu) when every
// valid cell of the pair starts on a table row (a re-seed row r H inside the table's row range
// and column window); returns false otherwise (the caller computes the seeds directly).
template <int DL, int G>
__device__ __forceinline__ bool seed_pair_tab(const MainParams& p, int g, long long delta0, bool ok0, bool ok1,
                                              long long row0, long long row1, __half2 (&QT)[DL]) {
    if (p.seed_tab == nullptr) return false;
    const __half* tab = reinterpret_cast<const __half*>(p.seed_tab);
    const long long row[2] = {row0, row1};
    const bool ok[2] = {ok0, ok1};
    long long base[2] = {0, 0};
#pragma unroll
    for (int u = 0; u < 2; ++u) {
        if (!ok[u]) continue;
        if (row[u] % p.H != 0) return false;
        const long long r = row[u] / p.H, j = row[u] + delta0 + u;
        if (r < p.tab_r_lo || r >= p.tab_r_hi || j < p.tab_j_lo || j >= p.tab_j_lo + p.tab_ldj) return false;
        base[u] = (r - p.tab_r_lo) * p.d * p.tab_ldj + (j - p.tab_j_lo);
    }
#pragma unroll
    for (int kk = 0; kk < DL; ++kk) {
        const int dim = kk * G + g;
        const bool pad = dim >= p.d;
        const __half h0 = pad ? __float2half(-1.f) : (ok0 ? tab[base[0] + (long long)dim * p.tab_ldj] : __float2half(0.f));
        const __half h1 = pad ? __float2half(-1.f) : (ok1 ? tab[base[1] + (long long)dim * p.tab_ldj] : __float2half(0.f));
        QT[kk] = __halves2half2(ok0 ? h0 : __low2half(QT[kk]), ok1 ? h1 : __high2half(QT[kk]));
    }
    return true;
}

template <int DL, int G, int NW, bool SELF, int MODE>
__global__ void __launch_bounds__(32 * NW, CtaShapeH<G>::MINB)
mp_diag_cta_h(const MainParams p) {
    using Cg = CtaGeoH<DL, G, NW>;
    using K = unsigned long long;
    using TS = typename std::conditional<fp32_precalc(MODE), float, __half>::type;  // seed operand type
    constexpr int D = Cg::D, NP = Cg::NP, NCC = Cg::NCC, RR = Cg::RR, RC = Cg::RC, SB = Cg::SB, NT = Cg::NT;
    static_assert(NP * G == NT, "G must divide the block");

    extern __shared__ __align__(16) unsigned char smem_raw[];
    H4* colv = reinterpret_cast<H4*>(smem_raw);
    RH* rowv = reinterpret_cast<RH*>(smem_raw + Cg::col_bytes);
    float* rowb = reinterpret_cast<float*>(smem_raw + Cg::col_bytes + Cg::row_bytes);
    float* colb = rowb + (size_t)RR * D;
    long long* tile_sh = reinterpret_cast<long long*>(smem_raw + Cg::col_bytes + Cg::row_bytes + Cg::stg_bytes);
    unsigned long long* bar = reinterpret_cast<unsigned long long*>(smem_raw + Cg::col_bytes + Cg::row_bytes + Cg::stg_bytes + 16);

    const RH* __restrict__ st_q = reinterpret_cast<const RH*>(p.st_q);   // row format [pos][dim]
    const H4* __restrict__ st_r = reinterpret_cast<const H4*>(p.st_r);   // pair format [pos + 1][dim]
    const TS* __restrict__ tw_q = reinterpret_cast<const TS*>(p.tw_q);
    const TS* __restrict__ tw_r = reinterpret_cast<const TS*>(p.tw_r);
    const TS* __restrict__ mu_q = reinterpret_cast<const TS*>(p.mu_q);
    const TS* __restrict__ mu_r = reinterpret_cast<const TS*>(p.mu_r);
    K* keys = reinterpret_cast<K*>(p.keys);

    const long long n = p.n;
    const int n32 = (int)n;
    const int d = p.d, m = p.m, H = p.H, HT = p.HT;
    const float two_mf = (float)(2 * m);
    const float FINF = __int_as_float(0x7f800000);
    const __half HZERO = __float2half(0.f), HINF = __ushort_as_half(0x7c00);
    const int tid = threadIdx.x;
    const int pp = tid / G, g = tid & (G - 1);  // cell pair of the block tile, lane within it

    // ring slot of a position: (pos + off) mod slots; off is a multiple of the slot count > n
    // so that column positions down to -1 (AB-join pairs starting at column -1) map to slots
    const int off_r = ((n32 + RR) / RR) * RR, off_c = ((n32 + RC) / RC) * RC;
    auto rslot = [&](int pos) { return (pos + off_r) % RR; };
    auto cslot = [&](int pos) { return (pos + off_c) % RC; };

    // TMA staging (MP_CTAH_TMA, d even so a position's d row entries of 8 B are whole 16-byte
    // units): one cp.async.bulk per entering position and side, issued by thread 0, completing
    // on the block's mbarrier (armed once per batch with the batch's byte count).  The padded
    // planes [d, D) of every slot never change and are written once; the thresholds still come
    // from the merge keys by cp.async and are converted after the batch (fixup).
    const bool tma = MP_CTAH_TMA && (d % 2) == 0;
    unsigned phase = 0;
    if (tma) {
        for (int e = tid; e < (RR + RC) * (D - d); e += NT) {
            const int sl = e / (D - d), pl = d + e % (D - d);
            if (sl < RR) {
                RH* dst = &rowv[sl * D + pl];
                dst->df = HZERO; dst->dg = HZERO; dst->a = HINF;
            } else {
                H4* dst = &colv[(sl - RR) * D + pl];
                dst->x = __half2half2(HZERO); dst->y = dst->x; dst->z = __half2half2(HINF);
            }
        }
        if (tid == 0) {
            mbar_init(bar, 1);
            fence_proxy_async();
        }
    }
    auto tma_issue = [&](int R0_, int r_lo, int r_hi, int C0_, int c_lo, int c_hi) {
        if (tid != 0) return;
        const unsigned rb = (unsigned)d * 8u, cb = (unsigned)d * 16u;
        unsigned bytes = 0;
        for (int q = r_lo; q < r_hi; ++q) bytes += rb;   // rows are always in range
        for (int q = c_lo; q < c_hi; ++q) {
            const int pos = C0_ + q;
            if (pos >= -1 && pos < n32) bytes += cb;
        }
        mbar_arrive_expect_tx(bar, bytes);
        for (int q = r_lo; q < r_hi; ++q) {
            const int pos = R0_ + q;
            bulk_g2s(&rowv[rslot(pos) * D], st_q + (size_t)pos * d, rb, bar);
        }
        for (int q = c_lo; q < c_hi; ++q) {
            const int pos = C0_ + q;
            if (pos >= -1 && pos < n32) bulk_g2s(&colv[cslot(pos) * D], st_r + (size_t)(pos + 1) * d, cb, bar);
        }
    };

    // stage positions [p_lo, p_hi) (relative to base) of one side: stats by cp.async (unless
    // TMA stages them), the threshold (value word of the merge key) into the float staging slot
    auto stage = [&](bool is_row, int base, int p_lo, int p_hi) {
        const int cnt = p_hi - p_lo;
        for (int e = tid; e < cnt * D; e += NT) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            const int rk = rank_of_plane<DL, G>(pl);
            if (is_row) {
                const int ix = rslot(pos) * D + pl;
                RH* dst = &rowv[ix];
                if (tma) {
                    // statistics by TMA (padded planes preset)
                } else if (pos >= 0 && pos < n32 && pl < d) {
                    cp_async8(dst, st_q + (size_t)pos * d + pl);      // (df, dg, a, -)
                } else {  // padded dimension / past the end: a = +inf with QT = -1 gives D = +inf
                    dst->df = HZERO; dst->dg = HZERO; dst->a = HINF;
                }
                if (pos >= 0 && pos < n32 && rk < d)
                    cp_async4(&rowb[ix], reinterpret_cast<const char*>(keys + (size_t)pos * d + rk) + 4);
                else
                    rowb[ix] = -FINF;  // never hit
            } else {
                const int ix = cslot(pos) * D + pl;
                H4* dst = &colv[ix];
                const bool in = pos >= -1 && pos < n32;
                if (in && pl < d) {
                    if (!tma) {
                        const H4* src = st_r + (size_t)(pos + 1) * d + pl;  // pair (pos, pos + 1)
                        cp_async8(dst, src);
                        cp_async4(&dst->z, &src->z);
                    }
                } else if (!(tma && in)) {   // TMA: padded planes of in-range positions are preset
                    dst->x = __half2half2(HZERO); dst->y = dst->x; dst->z = __half2half2(HINF);
                }
                if (SELF && pos >= 0 && pos < n32 && rk < d)
                    cp_async4(&colb[ix], reinterpret_cast<const char*>(keys + (size_t)pos * d + rk) + 4);
                else
                    colb[ix] = -FINF;
            }
        }
    };
    // after this thread's copies landed: half thresholds of the entries it staged (row -> .t;
    // column c -> low half of pair slot c and high half of pair slot c - 1)
    auto fixup = [&](bool is_row, int base, int p_lo, int p_hi) {
        const int cnt = p_hi - p_lo;
        for (int e = tid; e < cnt * D; e += NT) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            if (is_row) {
                const int ix = rslot(pos) * D + pl;
                rowv[ix].t = __float2half_rn(rowb[ix]);
            } else {
                const int ix = cslot(pos) * D + pl;
                const __half h = __float2half_rn(colb[ix]);
                reinterpret_cast<__half*>(&colv[ix].w)[0] = h;
                reinterpret_cast<__half*>(&colv[cslot(pos - 1) * D + pl].w)[1] = h;
            }
        }
    };

    for (;;) {
        if (tma) fence_proxy_async();   // this thread's generic ring writes precede later bulk copies
        __syncthreads();  // previous tile fully done (rings, tile_sh)
        if (tid == 0) *tile_sh = (long long)atomicAdd(p.counter, 1ull);
        __syncthreads();
        long long t = *tile_sh;
        if (t >= p.t_count) break;
        long long b, q;
        decode_tile(p, t, NCC, b, q);
        const long long delta0 = p.delta_lo + b * NCC;
        const long long delta1 = min(delta0 + NCC - 1, p.delta_hi);
        const long long rlo = max(0ll, -delta1), rhi = min(n, n - max(delta0, 0ll));
        const long long r0 = max(q * HT, rlo), r1 = min((q + 1) * HT, rhi);

        // this thread's pair: diagonals dP, dP + 1 and their valid rows [lo_u, hi_u)
        const long long dP = delta0 + 2 * pp;
        long long lo[2], hi[2];
        int lo32[2], hi32[2];
#pragma unroll
        for (int u = 0; u < 2; ++u) {
            lo[u] = max(r0, max(0ll, -(dP + u)));
            hi[u] = min(r1, n - max(dP + u, 0ll));
            if (dP + u > p.delta_hi) hi[u] = lo[u];
            lo32[u] = (int)lo[u];
            hi32[u] = (int)hi[u];
        }
        const int dP32 = (int)dP;

        __half2 QT[DL];
#pragma unroll
        for (int kk = 0; kk < DL; ++kk) QT[kk] = __float2half2_rn((kk * G + g) >= d ? -1.f : 0.f);
        // seeds: the tensor-core table (MP_SEEDS_TC) or direct dot products (FP16CK: compensated)
        // seeds: the tensor-core table (MODE 5) where the cell starts on a table row, else direct
        auto seed = [&](bool u0, bool u1, long long row0, long long row1) {
            if constexpr (MODE == 5)
                if (seed_pair_tab<DL, G>(p, g, dP, u0, u1, row0, row1, QT)) return;
            seed_pair_h<DL, G, MODE, TS>(tw_q, tw_r, mu_q, mu_r, m, d, g, dP, u0, u1, row0, row1, QT);
        };
        if (lo[0] < hi[0] || lo[1] < hi[1]) seed(lo[0] < hi[0], lo[1] < hi[1], lo[0], lo[1]);

        const int nrows = (int)(r1 - r0);
        const int R0 = (int)r0, C0 = (int)(r0 + delta0);  // row / first column of step 0
        // staged: rows [0, row_in), column positions [0, col_in) relative to R0 / C0; a batch
        // at s0 needs columns < s0 + SB + NCC - 1 (pair slots and their high thresholds)
        int row_in = min(SB, nrows), col_in = min(SB, nrows) + NCC;
        if (tma) tma_issue(R0, 0, row_in, C0, 0, col_in);
        stage(true, R0, 0, row_in);
        stage(false, C0, 0, col_in);
        cp_async_commit();
        cp_async_wait_all();
        if (tma) { mbar_wait(bar, phase); phase ^= 1; }
        fixup(true, R0, 0, row_in);
        fixup(false, C0, 0, col_in);
        __syncthreads();

        int seeded_step = -1;
        int to_seed = H;
        for (int s0 = 0; s0 < nrows; s0 += SB) {
            if (s0 > 0 && (to_seed -= SB) == 0) {  // re-seed the current row every H rows
                to_seed = H;
                const long long row = R0 + s0;
                const bool u0 = row > lo[0] && row < hi[0], u1 = row > lo[1] && row < hi[1];
                if (u0 || u1) seed(u0, u1, row, row);
                seeded_step = s0;
            }
            const int nxt = min(s0 + 2 * SB, nrows);
            const int r_lo = row_in, c_lo = col_in;
            if (tma) tma_issue(R0, row_in, max(row_in, nxt), C0, col_in, max(col_in, nxt + NCC));
            stage(true, R0, row_in, nxt);
            stage(false, C0, col_in, nxt + NCC);
            row_in = max(row_in, nxt);
            col_in = max(col_in, nxt + NCC);
            cp_async_commit();
            const int s1 = min(s0 + SB, nrows);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                const int row = R0 + s, cP = row + dP32;   // first column of the pair
                const int sr = rslot(row), sc = cslot(cP);
                bool active[2], upd[2];
#pragma unroll
                for (int u = 0; u < 2; ++u) {
                    active[u] = row >= lo32[u] && row < hi32[u];
                    upd[u] = row > lo32[u] && row < hi32[u] && s != seeded_step;
                }
                __half2 S[DL], th[DL];
                if (upd[0] == upd[1]) {
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) {
                        const int pl = kk * G + g;
                        const RH R = rowv[sr * D + pl];
                        const H4 C = colv[sc * D + pl];
                        if (upd[0]) QT[kk] = __hfma2(__half2half2(R.df), C.y, __hfma2(C.x, __half2half2(R.dg), QT[kk]));  // Eq. (1)
                        S[kk] = dist_pair(QT[kk], __hmul2(__half2half2(R.a), C.z), two_mf);     // Eq. (1)
                        th[kk] = SELF ? __hmax2(__half2half2(R.t), C.w) : __half2half2(R.t);
                    }
                } else {  // the two cells are at different phases (diagonal start / tile start)
                    const __half2 msk = __halves2half2(__float2half(upd[0] ? 1.f : 0.f), __float2half(upd[1] ? 1.f : 0.f));
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) {
                        const int pl = kk * G + g;
                        const RH R = rowv[sr * D + pl];
                        const H4 C = colv[sc * D + pl];
                        QT[kk] = __hfma2(msk, __hfma2(__half2half2(R.df), C.y, __hmul2(C.x, __half2half2(R.dg))), QT[kk]);
                        S[kk] = dist_pair(QT[kk], __hmul2(__half2half2(R.a), C.z), two_mf);
                        th[kk] = SELF ? __hmax2(__half2half2(R.t), C.w) : __half2half2(R.t);
                    }
                }
                sort_net<__half2, DL>(S);                                                // Eq. (2)
                if constexpr (MP_FUSE_LAST) {
                    lane_merge<__half2, DL, G, true>(S, g);
                    pair_scan<__half2, DL>(S);                                          // Eq. (2) scan
                } else {
                lane_merge<__half2, DL, G>(S, g);
                if constexpr (DL >= 8) {  // Eq. (2) inclusive scan, two half chains joined
#pragma unroll
                    for (int kk = 1; kk < DL / 2; ++kk) S[kk] = __hadd2(S[kk], S[kk - 1]);
#pragma unroll
                    for (int kk = DL / 2 + 1; kk < DL; ++kk) S[kk] = __hadd2(S[kk], S[kk - 1]);
#pragma unroll
                    for (int kk = DL / 2; kk < DL; ++kk) S[kk] = __hadd2(S[kk], S[DL / 2 - 1]);
                } else {
#pragma unroll
                    for (int kk = 1; kk < DL; ++kk) S[kk] = __hadd2(S[kk], S[kk - 1]);
                }
                }
                {
                    __half2 tot = S[DL - 1];
#pragma unroll
                    for (int dd = 1; dd < G; dd <<= 1) {
                        const __half2 y = __shfl_up_sync(FULL, tot, dd, G);
                        if (g >= dd) tot = __hadd2(tot, y);
                    }
                    __half2 excl = __shfl_up_sync(FULL, tot, 1, G);
                    if (g == 0) excl = __float2half2_rn(0.f);
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) S[kk] = __hadd2(S[kk], excl);
                }
                const unsigned act = (active[0] ? 0x0000ffffu : 0u) | (active[1] ? 0xffff0000u : 0u);
                unsigned hm[4] = {0u, 0u, 0u, 0u};
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) hm[kk & 3] |= __hle2_mask(S[kk], th[kk]);
                if (((hm[0] | hm[1]) | (hm[2] | hm[3])) & act) {
                    // Eq. (3), lane-local: merge (value, index) keys straight into global memory
                    // and lower the ring's threshold hints
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) {
                        const unsigned mk = __hle2_mask(S[kk], th[kk]) & act;
                        if (mk == 0u) continue;
                        const int pl = kk * G + g;
                        const int rk = g * DL + kk;  // rank held in register kk after the merge
#pragma unroll
                        for (int u = 0; u < 2; ++u) {
                            if ((mk & (u ? 0xffff0000u : 0x0000ffffu)) == 0u) continue;
                            const __half hv = u ? __high2half(S[kk]) : __low2half(S[kk]);
                            const float v = __half2float(hv);
                            const unsigned vb = __float_as_uint(v);
                            const int col = cP + u;
                            RH* rp = &rowv[sr * D + pl];
                            const float tr = __half2float(rp->t);
                            if (v <= tr) {
                                atomicMin(keys + (size_t)row * d + rk, ((K)vb << 32) | (unsigned)col);
                                if (v < tr) atomic_min_half(&rp->t, hv);
                            }
                            if (SELF) {
                                __half* cw = reinterpret_cast<__half*>(&colv[cslot(col) * D + pl].w);
                                const float tc = __half2float(cw[0]);
                                if (v <= tc) {
                                    atomicMin(keys + (size_t)col * d + rk, ((K)vb << 32) | (unsigned)row);
                                    if (v < tc) {
                                        atomic_min_half(&cw[0], hv);
                                        atomic_min_half(&reinterpret_cast<__half*>(&colv[cslot(col - 1) * D + pl].w)[1], hv);
                                    }
                                }
                            }
                        }
                    }
                }
            }
            cp_async_wait_all();               // this thread's prefetch landed ...
            if (tma) { mbar_wait(bar, phase); phase ^= 1; }   // ... and the batch's bulk copies
            fixup(true, R0, r_lo, row_in);     // ... so it converts the thresholds it staged
            fixup(false, C0, c_lo, col_in);
            if (tma) fence_proxy_async();      // generic ring accesses before the next bulk copies
            __syncthreads();                   // publish; this batch's reads are all done
        }
    }
}

template <int DL, int G, int NW, bool SELF, int MODE> struct InstCtaH {
    static size_t smem() { return CtaGeoH<DL, G, NW>::bytes; }
    static cudaError_t launch(const MainParams& p, int grid, cudaStream_t s);
    static int blocks_per_sm();
};

#ifdef MP_DIAG_IMPL
template <int DL, int G, int NW, bool SELF, int MODE>
cudaError_t InstCtaH<DL, G, NW, SELF, MODE>::launch(const MainParams& p, int grid, cudaStream_t s) {
    const size_t sm = smem();
    cudaError_t e = cudaFuncSetAttribute(mp_diag_cta_h<DL, G, NW, SELF, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    mp_diag_cta_h<DL, G, NW, SELF, MODE><<<grid, 32 * NW, sm, s>>>(p);
    return cudaGetLastError();
}
template <int DL, int G, int NW, bool SELF, int MODE> int InstCtaH<DL, G, NW, SELF, MODE>::blocks_per_sm() {
    const size_t sm = smem();
    cudaFuncSetAttribute(mp_diag_cta_h<DL, G, NW, SELF, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    int nb = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, mp_diag_cta_h<DL, G, NW, SELF, MODE>, 32 * NW, sm);
    return nb;
}
#endif

}  // namespace mpk

#pragma once
// mp_diag16.cuh -- the fused diagonal kernel in half precision (FP16, Mixed and FP16C modes,
// PAPER.md Fig. 1 table, Sec. III-C: "FP16 for storage and computation";
// Mixed differs in a FP32 precalculation, FP16C in compensated half sums).
//
// Same structure as mp_diag (mp_diag.cuh): warp tiles of consecutive diagonals, staggered
// lane-cells, per-warp shared-memory rings staged by cp.async one batch ahead, filtered
// min/argmin with a warp-shuffle slow path.  Differences:
//   * a lane-cell is a PAIR of adjacent diagonals (delta, delta+1) packed into __half2, so
//     every FMA / min / max / compare of the main loop processes two cells (HFMA2, HMNMX2);
//   * row ring entries are 8 B (df, dg, a, threshold as halves; the .H0_H0 operand swizzle
//     broadcasts them to both cells for free); column ring entries hold the pair
//     (x_c, x_{c+1}) (precomputed in global memory), so one LDS.128 feeds both cells;
//   * every running best is a half value, so the ring's half threshold IS the best: the slow
//     path compares against it and writes improvements straight through to the global merge
//     key (RED.MIN.64 on (float bits << 32 | j), which also applies the lowest-index tie
//     rule); there is no eviction pass.  Thresholds enter the ring through a 4 B float
//     staging slot (cp.async of the key's value word) converted once the copy has landed.
// Keys, finalize and the multi-GPU merge are the FP32 ones (float bits << 32 | j).
#include <cuda_fp16.h>
#include <type_traits>
#include "mp_diag.cuh"

namespace mpk {

// Lower a non-negative half-precision threshold hint towards v with ONE 32-bit atomicMin on the
// word holding it (non-negative halves order as their bits; the word's other half is re-used as
// read).  If the other half was lowered concurrently the atomic may skip this update or restore
// the other half's older, higher value: a hint can end up higher than the best -- an extra
// slow-path visit -- but never lower, and never torn.  Plain loads by other lanes always see a
// value that was merged into the global keys.
__device__ __forceinline__ void atomic_min_half(__half* p, __half v) {   // p: shared memory
    const unsigned sa = (unsigned)__cvta_generic_to_shared(p);
    const unsigned wa = sa & ~3u;
    const bool hi = (sa & 2u) != 0;
    unsigned old;
    asm volatile("ld.volatile.shared.u32 %0, [%1];" : "=r"(old) : "r"(wa) : "memory");
    const unsigned hv = __half_as_ushort(v);
    const unsigned nw = hi ? ((hv << 16) | (old & 0xffffu)) : ((old & 0xffff0000u) | hv);
    asm volatile("red.shared.min.u32 [%0], %1;" ::"r"(wa), "r"(nw) : "memory");
}

template <> struct PT<__half2> {
    static __device__ __forceinline__ __half2 vmin(__half2 a, __half2 b) { return __hmin2(a, b); }
    static __device__ __forceinline__ __half2 vmax(__half2 a, __half2 b) { return __hmax2(a, b); }
};

// D of a cell pair (Eq. 1): D^2 = 2m - QT (a_i a_j) by a mixed-precision FMA (half operands,
// FP32 result: FHFMA, .H0/.H1 selectors, no half rounding of D^2 and no conversion before the
// FP32 square root), then sqrt of |D^2| (reading G5) rounded to half (reading G14).
__device__ __forceinline__ __half2 dist_pair(__half2 qt, __half2 aa, float two_m) {
    float lo, hi;
    asm("{\n .reg .f16 q0, q1, a0, a1;\n mov.b32 {q0, q1}, %2;\n mov.b32 {a0, a1}, %3;\n"
        " neg.f16 q0, q0;\n neg.f16 q1, q1;\n"
        " fma.rn.f32.f16 %0, q0, a0, %4;\n fma.rn.f32.f16 %1, q1, a1, %4;\n}"
        : "=f"(lo), "=f"(hi)
        : "r"(*reinterpret_cast<const unsigned*>(&qt)), "r"(*reinterpret_cast<const unsigned*>(&aa)), "f"(two_m));
    float slo, shi;
    asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(slo) : "f"(fabsf(lo)));
    asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(shi) : "f"(fabsf(hi)));
    return __floats2half2_rn(slo, shi);
}

struct alignas(8) RH { __half df, dg, a, t; };   // row ring entry (one position)
struct alignas(16) H4 { __half2 x, y, z, w; };   // column ring entry (pair c, c+1)

// warps per block (1..4) that maximise resident warps per SM under the shared-memory budget
// (228 KB per SM, 1 KB reserved per block, 227 KB per block, 32 blocks per SM)
constexpr int best_wpb(size_t bpw) {
    int best = 1, bw = 0;
    for (int w = 1; w <= 4; ++w) {
        if (bpw * w > 227u * 1024u) break;
        int nb = (int)((228u * 1024u) / (bpw * w + 1024u));
        if (nb > 32) nb = 32;
        if (nb * w >= bw) { bw = nb * w; best = w; }
    }
    return best;
}

template <int DL, int G> struct SmemH {
    using Gm = Geo<G, 2>;
    static constexpr int D = DL * G;
    static constexpr size_t a16(size_t x) { return (x + 15) & ~(size_t)15; }
    static constexpr size_t col_bytes = (size_t)D * Gm::PSC * sizeof(H4);
    static constexpr size_t row_bytes = a16((size_t)D * Gm::PSR * sizeof(RH));
    static constexpr size_t thr_bytes = a16((size_t)D * (Gm::PSR + Gm::PSC) * sizeof(float));
    static constexpr size_t bytes_per_warp = col_bytes + row_bytes + thr_bytes + (size_t)DL * 32 * sizeof(__half2);
    static constexpr int WPB = best_wpb(bytes_per_warp);
};

// DL operands of plane kk*G + g from a position-major row (vector loads when G == 1)
template <class T, int DL, int G>
__device__ __forceinline__ void ldv(const T* __restrict__ rowp, int g, T (&out)[DL]) {
    constexpr int PER = 16 / (int)sizeof(T);
    if constexpr (G == 1 && DL % PER == 0) {
#pragma unroll
        for (int q = 0; q < DL / PER; ++q) {
            const uint4 v = __ldg(reinterpret_cast<const uint4*>(rowp) + q);
            const T* e = reinterpret_cast<const T*>(&v);
#pragma unroll
            for (int r = 0; r < PER; ++r) out[q * PER + r] = e[r];
        }
    } else {
#pragma unroll
        for (int kk = 0; kk < DL; ++kk) out[kk] = rowp[kk * G + g];
    }
}

// Seeds of one cell pair (diagonals delta0, delta0 + 1): direct centred dot products
// (reading G8) at rows row0 / row1 (cells with ok_u false keep their QT).
// Mixed -> FP32 operands and accumulation rounded to half (the FP32 precalc; FP16CK: with Kahan
// compensation, the text's FP16C reading L786-791); FP16 -> half arithmetic;
// FP16C -> half arithmetic with Kahan compensation (Fig. 1 reading).  When both cells start on the
// same row the row window is shared and the second column window is the first shifted by one.
// Half-kernel modes: 0 FP16, 1 Mixed, 2 FP16C (Fig. 1), 3 FP16CK (the text's FP16C: Mixed with
// Kahan-compensated FP32 seeds), 5 Mixed / FP16CK reading the tensor-core seed table (block kernel)
constexpr bool fp32_precalc(int mode) { return mode == 1 || mode == 3 || mode == 5; }

template <int DL, int G, int MODE, class TS>
__device__ __forceinline__ void seed_pair_h(const TS* __restrict__ tw_q, const TS* __restrict__ tw_r,
                                            const TS* __restrict__ mu_q, const TS* __restrict__ mu_r,
                                            int m, int d, int g, long long delta0, bool ok0, bool ok1,
                                            long long row0, long long row1, __half2 (&QT)[DL]) {
    constexpr int D = DL * G;
    const long long delta[2] = {delta0, delta0 + 1};
    using TA = TS;
    const bool same = ok0 && ok1 && row0 == row1;
    TA acc0[DL], acc1[DL];
#pragma unroll
    for (int kk = 0; kk < DL; ++kk) { acc0[kk] = (TA)0.f; acc1[kk] = (TA)0.f; }
    constexpr bool comp = MODE == 2 || MODE == 3;
    auto kadd = [](TA& acc, TA& cp, TA v) {
        if constexpr (comp) {  // compensated accumulation
            const TA y = v - cp;
            const TA t2 = acc + y;
            cp = (t2 - acc) - y;
            acc = t2;
        } else {
            acc = acc + v;
        }
    };
    // dims in chunks of one 16-byte vector per operand: the m-long loop keeps few
    // operand registers live, so seeding does not set the kernel's register peak
    constexpr int SC = (16 / (int)sizeof(TA)) < DL ? (16 / (int)sizeof(TA)) : DL;
    if (same) {
        const long long i0 = row0, j0 = row0 + delta[0];
#pragma unroll
        for (int c0 = 0; c0 < DL; c0 += SC) {
            TA mq[SC], mr0[SC], mr1[SC], xr[SC], a0[SC], a1[SC], k0[SC], k1[SC];
            ldv<TA, SC, G>(mu_q + i0 * D + c0 * G, g, mq);
            ldv<TA, SC, G>(mu_r + j0 * D + c0 * G, g, mr0);
            ldv<TA, SC, G>(mu_r + (j0 + 1) * D + c0 * G, g, mr1);
            ldv<TA, SC, G>(tw_r + j0 * D + c0 * G, g, xr);
#pragma unroll
            for (int kk = 0; kk < SC; ++kk) { a0[kk] = (TA)0.f; a1[kk] = (TA)0.f; k0[kk] = (TA)0.f; k1[kk] = (TA)0.f; }
#pragma unroll 4
            for (int tt = 0; tt < m; ++tt) {
                TA xq[SC], xn[SC];
                ldv<TA, SC, G>(tw_q + (i0 + tt) * D + c0 * G, g, xq);
                ldv<TA, SC, G>(tw_r + (j0 + tt + 1) * D + c0 * G, g, xn);   // j0 + m <= L - 1 (cell 1 valid)
#pragma unroll
                for (int kk = 0; kk < SC; ++kk) {
                    const TA cq = xq[kk] - mq[kk];
                    kadd(a0[kk], k0[kk], cq * (xr[kk] - mr0[kk]));
                    kadd(a1[kk], k1[kk], cq * (xn[kk] - mr1[kk]));
                    xr[kk] = xn[kk];
                }
            }
#pragma unroll
            for (int kk = 0; kk < SC; ++kk) { acc0[c0 + kk] = a0[kk]; acc1[c0 + kk] = a1[kk]; }
        }
    } else {
#pragma unroll 1
        for (int u = 0; u < 2; ++u) {
            if (!(u == 0 ? ok0 : ok1)) continue;
            const long long i0 = u == 0 ? row0 : row1, j0 = i0 + delta[u];
#pragma unroll
            for (int c0 = 0; c0 < DL; c0 += SC) {
                TA mq[SC], mr[SC], acc[SC], cp[SC];
                ldv<TA, SC, G>(mu_q + i0 * D + c0 * G, g, mq);
                ldv<TA, SC, G>(mu_r + j0 * D + c0 * G, g, mr);
#pragma unroll
                for (int kk = 0; kk < SC; ++kk) { acc[kk] = (TA)0.f; cp[kk] = (TA)0.f; }
#pragma unroll 4
                for (int tt = 0; tt < m; ++tt) {
                    TA xq[SC], xr[SC];
                    ldv<TA, SC, G>(tw_q + (i0 + tt) * D + c0 * G, g, xq);
                    ldv<TA, SC, G>(tw_r + (j0 + tt) * D + c0 * G, g, xr);
#pragma unroll
                    for (int kk = 0; kk < SC; ++kk) kadd(acc[kk], cp[kk], (xq[kk] - mq[kk]) * (xr[kk] - mr[kk]));
                }
#pragma unroll
                for (int kk = 0; kk < SC; ++kk) { if (u == 0) acc0[c0 + kk] = acc[kk]; else acc1[c0 + kk] = acc[kk]; }
            }
        }
    }
#pragma unroll
    for (int kk = 0; kk < DL; ++kk) {
        const bool pad = (kk * G + g) >= d;
        const __half h0 = __float2half_rn(pad ? -1.f : (float)acc0[kk]);
        const __half h1 = __float2half_rn(pad ? -1.f : (float)acc1[kk]);
        QT[kk] = __halves2half2(ok0 ? h0 : __low2half(QT[kk]), ok1 ? h1 : __high2half(QT[kk]));
    }
}

// MODE: 0 = FP16, 1 = Mixed (FP32 precalc and seeds), 2 = FP16C (half precalc and seeds with
// Kahan-compensated sums, reading G17)
template <int DL, int G, bool SELF, int MODE>
__global__ void __launch_bounds__(128)
mp_diag_h(const MainParams p) {
    constexpr bool MIXED = fp32_precalc(MODE);
    using Gm = Geo<G, 2>;
    using SM = SmemH<DL, G>;
    using TS = typename std::conditional<MIXED, float, __half>::type;  // seed operand type
    constexpr int CA = Gm::CA, RA = Gm::RA, CW = Gm::CW, D = DL * G;
    constexpr int PSR = Gm::PSR, PSC = Gm::PSC, SB = Gm::SB;

    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned char* wbase = smem_raw + (size_t)warp * SM::bytes_per_warp;
    H4* colv = reinterpret_cast<H4*>(wbase);
    RH* rowv = reinterpret_cast<RH*>(wbase + SM::col_bytes);
    float* rowb = reinterpret_cast<float*>(wbase + SM::col_bytes + SM::row_bytes);
    float* colb = rowb + (size_t)D * PSR;
    __half2* ssc = reinterpret_cast<__half2*>(wbase + SM::col_bytes + SM::row_bytes + SM::thr_bytes);

    const RH* __restrict__ st_q = reinterpret_cast<const RH*>(p.st_q);   // row format
    const H4* __restrict__ st_r = reinterpret_cast<const H4*>(p.st_r);   // pair format (x_c, x_c+1)
    const TS* __restrict__ tw_q = reinterpret_cast<const TS*>(p.tw_q);
    const TS* __restrict__ tw_r = reinterpret_cast<const TS*>(p.tw_r);
    const TS* __restrict__ mu_q = reinterpret_cast<const TS*>(p.mu_q);
    const TS* __restrict__ mu_r = reinterpret_cast<const TS*>(p.mu_r);
    unsigned long long* keys = reinterpret_cast<unsigned long long*>(p.keys);

    const long long n = p.n;
    const int d = p.d, m = p.m, H = p.H, HT = p.HT;
    const int n32 = (int)n;
    const float two_mf = (float)(2 * m);
    const float FINF = __int_as_float(0x7f800000);
    const __half HZERO = __float2half(0.f), HINF = __ushort_as_half(0x7c00);

    const int lc = lane >> Gm::LOG_G, g = lane & (G - 1);
    const int a = lc >> Gm::LOG_CA, c = lc & (CA - 1);
    unsigned gmask_row = 0, gmask_col = 0;
#pragma unroll
    for (int cc = 0; cc < CA; ++cc) gmask_row |= 1u << (((a * CA + cc) << Gm::LOG_G) + g);
#pragma unroll
    for (int aa = 0; aa < RA; ++aa) gmask_col |= 1u << (((aa * CA + c) << Gm::LOG_G) + g);

    // ---- staging: stats by cp.async, the key's value word into the float staging slot;
    // fixup() writes the half thresholds once the copies have landed.  Column pairs start
    // at position -1 (the pair (-1, 0) feeds cells whose first column is 0).
    auto stage = [&](bool is_row, int base, int p_lo, int p_hi) {
        const int cnt = p_hi - p_lo;
        if (cnt <= 0) return;
        float* bb = is_row ? rowb : colb;
        const int ps = is_row ? PSR : PSC;
        const bool want_thr = is_row || SELF;
        for (int e = lane; e < cnt * D; e += 32) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            if (pos < (is_row ? 0 : -1) || pos >= n32) continue;
            const int sl = is_row ? Gm::srow(pos) : Gm::scol(pos);
            if (is_row) {
                RH* dst = &rowv[pl * PSR + sl];
                if (pl < d) {
                    cp_async8(dst, st_q + (size_t)pos * d + pl);        // (df, dg, a, -)
                } else {  // padded dimension: a = +inf with QT = -1 gives D = +inf
                    dst->df = HZERO; dst->dg = HZERO; dst->a = HINF;
                }
            } else {
                H4* dst = &colv[pl * PSC + sl];
                if (pl < d) {
                    const H4* src = st_r + (size_t)(pos + 1) * d + pl;
                    cp_async8(dst, src);
                    cp_async4(&dst->z, &src->z);
                } else {
                    dst->x = __half2half2(HZERO); dst->y = dst->x; dst->z = __half2half2(HINF);
                }
            }
            const int rk = rank_of_plane<DL, G>(pl);
            if (rk < d && want_thr && pos >= 0)
                cp_async4(&bb[pl * ps + sl], reinterpret_cast<const char*>(keys + (size_t)pos * d + rk) + 4);
            else
                bb[pl * ps + sl] = -FINF;  // never hit
        }
    };
    // half thresholds from the landed values (exact: every stored best is a half value):
    // row -> .t; column c -> low half of slot c and high half of slot c-1 (the pair (c-1, c))
    auto fixup = [&](bool is_row, int base, int p_lo, int p_hi) {
        const int cnt = p_hi - p_lo;
        if (cnt <= 0) return;
        for (int e = lane; e < cnt * D; e += 32) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            if (pos < (is_row ? 0 : -1) || pos >= n32) continue;
            if (is_row) {
                const int ix = pl * PSR + Gm::srow(pos);
                rowv[ix].t = __float2half_rn(rowb[ix]);
            } else {
                const int ix = pl * PSC + Gm::scol(pos);
                const __half h = __float2half_rn(colb[ix]);
                reinterpret_cast<__half*>(&colv[ix].w)[0] = h;
                if (pos >= 0) reinterpret_cast<__half*>(&colv[pl * PSC + Gm::scol(pos - 1)].w)[1] = h;
            }
        }
    };

    for (;;) {
        long long t = 0;
        if (lane == 0) t = (long long)atomicAdd(p.counter, 1ull);
        t = __shfl_sync(FULL, t, 0);
        if (t >= p.t_count) break;
        long long b, q;
        decode_tile(p, t, Gm::NC, b, q);
        const long long delta0 = p.delta_lo + b * Gm::NC;
        const long long delta1 = min(delta0 + Gm::NC - 1, p.delta_hi);
        const long long rlo = max(0ll, -delta1), rhi = min(n, n - max(delta0, 0ll));
        const long long r0 = max(q * HT, rlo), r1 = min((q + 1) * HT, rhi);

        long long delta[2], lo[2], hi[2];
        int dlt[2], lo32[2], hi32[2];
#pragma unroll
        for (int u = 0; u < 2; ++u) {
            delta[u] = delta0 + (long long)a * CW + c * 2 + u;
            lo[u] = max(r0, max(0ll, -delta[u]));
            hi[u] = min(r1, n - max(delta[u], 0ll));
            if (delta[u] > p.delta_hi) hi[u] = lo[u];
            dlt[u] = (int)delta[u]; lo32[u] = (int)lo[u]; hi32[u] = (int)hi[u];
        }

        __half2 QT[DL];
        auto seed_pair = [&](bool ok0, bool ok1, long long row0, long long row1) {
            seed_pair_h<DL, G, MODE, TS>(tw_q, tw_r, mu_q, mu_r, m, d, g, delta[0], ok0, ok1, row0, row1, QT);
        };
#pragma unroll
        for (int kk = 0; kk < DL; ++kk) QT[kk] = __float2half2_rn((kk * G + g) >= d ? -1.f : 0.f);
        int seeded_step = -1;

        const int nrows = (int)(r1 - r0);
        const int s_end = nrows + CW * (RA - 1);
        const int R0 = (int)r0, C0 = (int)(r0 + delta0);
        int row_in = min(SB, nrows), col_in = min(SB, s_end) + CW;  // pairs need column c+1's slot too
        int fx_r0 = 0, fx_c0 = 0;
        stage(true, R0, 0, row_in);
        stage(false, C0, 0, col_in);
        cp_async_commit();
        cp_async_wait_all();
        __syncwarp();
        fixup(true, R0, 0, row_in);
        fixup(false, C0, 0, col_in);
        fx_r0 = row_in; fx_c0 = col_in;
        __syncwarp();

        auto step = [&](int s) {
            const int row = R0 + s - CW * a;
            const int sr = Gm::srow(row);
            const int col0 = row + dlt[0];
            const int scn = Gm::scol(col0);
            bool active[2], upd[2];
#pragma unroll
            for (int u = 0; u < 2; ++u) {
                active[u] = row >= lo32[u] && row < hi32[u];
                upd[u] = row > lo32[u] && row < hi32[u];
            }
            if (s == seeded_step) upd[0] = upd[1] = false;  // QT of this row was just seeded
            // D (Eq. 1) for both cells; threshold = max of the row's and the column's best
            // (a cell can improve either iff S_k <= that max)
            __half2 S[DL], th[DL];
            if (upd[0] == upd[1]) {
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    const int pl = kk * G + g;
                    const RH R = rowv[pl * PSR + sr];
                    const H4 C = colv[pl * PSC + scn];
                    if (upd[0]) QT[kk] = __hfma2(__half2half2(R.df), C.y, __hfma2(C.x, __half2half2(R.dg), QT[kk]));
                    S[kk] = dist_pair(QT[kk], __hmul2(__half2half2(R.a), C.z), two_mf);
                    th[kk] = SELF ? __hmax2(__half2half2(R.t), C.w) : __half2half2(R.t);
                }
            } else {  // the two cells of the pair are at different phases (tile / diagonal start)
                const __half2 msk = __halves2half2(__float2half(upd[0] ? 1.f : 0.f), __float2half(upd[1] ? 1.f : 0.f));
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    const int pl = kk * G + g;
                    const RH R = rowv[pl * PSR + sr];
                    const H4 C = colv[pl * PSC + scn];
                    QT[kk] = __hfma2(msk, __hfma2(__half2half2(R.df), C.y, __hmul2(C.x, __half2half2(R.dg))), QT[kk]);
                    S[kk] = dist_pair(QT[kk], __hmul2(__half2half2(R.a), C.z), two_mf);
                    th[kk] = SELF ? __hmax2(__half2half2(R.t), C.w) : __half2half2(R.t);
                }
            }
            sort_net<__half2, DL>(S);                                              // Eq. (2)
            if (G > 1) lane_merge<__half2, DL, G>(S, g);
            // Eq. (2) inclusive scan, two independent half chains joined at the end (shorter
            // dependency chain; the summation order differs only by rounding)
            if constexpr (DL >= 8) {
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
            if (G > 1) {
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
            unsigned hm[4] = {0u, 0u, 0u, 0u};
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) hm[kk & 3] |= __hle2_mask(S[kk], th[kk]);
            const unsigned hmask = (hm[0] | hm[1]) | (hm[2] | hm[3]);
            const bool hit = ((hmask & 0xffffu) && active[0]) || ((hmask >> 16) && active[1]);
            if (__any_sync(FULL, hit)) {
                // Eq. (3): group min by shuffles; the leader of a row / column group compares
                // with the ring's best and writes an improvement (or a tie, for the index
                // rule) through to the merge key.
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    __half2 v = S[kk];
                    if (!active[0]) v = __halves2half2(HINF, __high2half(v));
                    if (!active[1]) v = __halves2half2(__low2half(v), HINF);
                    ssc[kk * 32 + lane] = v;
                }
                // ranks some lane can improve (a superset: staged thresholds only decrease);
                // the loop then visits only those -- a slow step typically touches 1-2 ranks
                const unsigned act = (active[0] ? 0x0000ffffu : 0u) | (active[1] ? 0xffff0000u : 0u);
                unsigned rk_bits = 0;
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) rk_bits |= (unsigned)((__hle2_mask(S[kk], th[kk]) & act) != 0u) << kk;
                rk_bits = __reduce_or_sync(FULL, rk_bits);
                __syncwarp();
#pragma unroll 1
                for (; rk_bits != 0; rk_bits &= rk_bits - 1) {
                    const int kk = __ffs(rk_bits) - 1;
                    const int pl = kk * G + g;
                    const int rk = g * DL + kk;  // rank held in register kk after the merge
                    const __half2 vh = ssc[kk * 32 + lane];
                    const float v[2] = {__low2float(vh), __high2float(vh)};
                    const int ixr = pl * PSR + sr;
                    const float tr = __half2float(rowv[ixr].t);
                    float tc[2] = {-FINF, -FINF};
                    if (SELF) {
                        const __half2 w = colv[pl * PSC + scn].w;
                        tc[0] = __low2float(w);
                        tc[1] = __high2float(w);
                    }
                    const bool need_r = __any_sync(FULL, fminf(v[0], v[1]) <= tr);
                    const bool need_c = SELF && __any_sync(FULL, v[0] <= tc[0] || v[1] <= tc[1]);
                    __syncwarp();   // every lane read the hints before a leader lowers them
                    if (need_r) {
                        float vr = fminf(v[0], v[1]);
#pragma unroll
                        for (int bit = 0; bit < Gm::LOG_CA; ++bit)
                            vr = fminf(vr, __shfl_xor_sync(FULL, vr, 1 << (bit + Gm::LOG_G)));
                        const unsigned eqr = __ballot_sync(FULL, v[0] == vr || v[1] == vr) & gmask_row;
                        if (vr < FINF && vr <= tr && lane == __ffs(eqr) - 1) {
                            const int j = (v[0] == vr) ? col0 : col0 + 1;          // lowest column first
                            KeyOps<float>::merge(keys + (size_t)row * d + rk, vr, (unsigned)j);
                            if (vr < tr) atomic_min_half(&rowv[ixr].t, __float2half_rn(vr));   // exact
                        }
                    }
                    if (SELF && need_c) {
#pragma unroll
                        for (int u = 0; u < 2; ++u) {
                            float vc = v[u];
#pragma unroll
                            for (int bit = 0; bit < 5 - Gm::LOG_G - Gm::LOG_CA; ++bit)
                                vc = fminf(vc, __shfl_xor_sync(FULL, vc, 1 << (bit + Gm::LOG_G + Gm::LOG_CA)));
                            const unsigned eqc = __ballot_sync(FULL, v[u] == vc) & gmask_col;
                            // lowest row index = highest a = highest lane
                            if (vc < FINF && vc <= tc[u] && eqc != 0 && lane == 31 - __clz(eqc)) {
                                const int colu = col0 + u;
                                KeyOps<float>::merge(keys + (size_t)colu * d + rk, vc, (unsigned)row);
                                if (vc < tc[u]) {
                                    const __half h = __float2half_rn(vc);
                                    atomic_min_half(&reinterpret_cast<__half*>(&colv[pl * PSC + Gm::scol(colu)].w)[0], h);
                                    atomic_min_half(&reinterpret_cast<__half*>(&colv[pl * PSC + Gm::scol(colu - 1)].w)[1], h);
                                }
                            }
                        }
                    }
                    __syncwarp();   // the leaders' hint stores are visible to the next rank's reads
                }
                __syncwarp();
            }
        };

        int to_seed = SB;  // steps until the next seed (H is a multiple of SB)
        for (int s0 = 0; s0 < s_end; s0 += SB) {
            if ((to_seed -= SB) == 0) {  // seeds: first rows at s0 = 0, current row every H steps
                to_seed = H;
                const long long row = R0 + s0 - (long long)CW * a;
                if (s0 == 0) {
                    seed_pair(lo[0] < hi[0], lo[1] < hi[1], lo[0], lo[1]);
                } else {
                    const bool u0 = row > lo[0] && row < hi[0], u1 = row > lo[1] && row < hi[1];
                    if (u0 || u1) seed_pair(u0, u1, row, row);
                }
                seeded_step = s0 == 0 ? -1 : s0;
            }
            // prefetch the next batch's entries (positions older than this batch are dead:
            // the rings hold exactly the live span, bests were written through)
            const int nxt = min(s0 + 2 * SB, s_end);
            const int r_need = min(nxt, nrows), c_need = nxt + CW;
            stage(true, R0, row_in, r_need);
            stage(false, C0, col_in, c_need);
            const int fx_r1 = max(row_in, r_need), fx_c1 = max(col_in, c_need);
            row_in = fx_r1;
            col_in = fx_c1;
            cp_async_commit();
            const int s1 = min(s0 + SB, s_end);
#pragma unroll 1
            for (int ss = s0; ss < s1; ++ss) step(ss);
            cp_async_wait_all();
            __syncwarp();
            fixup(true, R0, fx_r0, fx_r1);
            fixup(false, C0, fx_c0, fx_c1);
            fx_r0 = fx_r1;
            fx_c0 = fx_c1;
            __syncwarp();
        }
        __syncwarp();
    }
}

template <int DL, int G, bool SELF, int MODE> struct InstH {
    static size_t smem() { return SmemH<DL, G>::bytes_per_warp * SmemH<DL, G>::WPB; }
    static int warps_per_block() { return SmemH<DL, G>::WPB; }
    static cudaError_t launch(const MainParams& p, int grid, cudaStream_t s);
    static int blocks_per_sm();
};

#ifdef MP_DIAG_IMPL
template <int DL, int G, bool SELF, int MODE>
cudaError_t InstH<DL, G, SELF, MODE>::launch(const MainParams& p, int grid, cudaStream_t s) {
    const size_t sm = smem();
    cudaError_t e = cudaFuncSetAttribute(mp_diag_h<DL, G, SELF, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    mp_diag_h<DL, G, SELF, MODE><<<grid, SmemH<DL, G>::WPB * 32, sm, s>>>(p);
    return cudaGetLastError();
}
template <int DL, int G, bool SELF, int MODE> int InstH<DL, G, SELF, MODE>::blocks_per_sm() {
    const size_t sm = smem();
    cudaFuncSetAttribute(mp_diag_h<DL, G, SELF, MODE>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    int nb = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, mp_diag_h<DL, G, SELF, MODE>, SmemH<DL, G>::WPB * 32, sm);
    return nb;
}
#endif

}  // namespace mpk

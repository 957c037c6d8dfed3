#pragma once
// mp_diag64f.cuh -- FP64 fused diagonal kernel with an FP32 filter.
//
// FP64 mode (Fig. 1: precalculation FP64, main loop FP64) computes the QT
// recurrence (Eq. 1) and D^2 = 2m - QT a_i a_j in FP64 for every cell.  Most cells cannot
// improve any profile entry, and deciding that does not need FP64: the sorted prefix sums
// S_k (Eq. 2) are formed in FP32 from D^2 rounded to FP32, and compared with FP32 copies of
// the running bests rounded UP and widened by a relative margin that bounds the FP32
// rounding of S (conservative: a cell that could improve an entry is never filtered out).
// A warp step where some lane passes the filter re-runs the exact FP64 path (FP64 sqrt,
// sort, scan) for all its cells and merges with the authoritative FP64 bests, exactly as
// the unfiltered kernel.  Results are identical to a pure FP64 evaluation of the same cells.
//
// Structure as mp_diag (mp_diag.cuh): warp tiles, staggered lane-cells, cp.async-staged
// per-warp rings (entries: df, dg, a in FP64 + the FP32 filter threshold).  The exact path
// writes through: a row / column group leader merges its (value, index) into the global
// merge key with a 128-bit CAS (lexicographic min, reading G2) and lowers the ring's
// threshold; the authoritative bests live only in global memory, which keeps the ring at
// 32 B per (position, dim) and the kernel at 8 resident warps per SM.
#include "mp_diag.cuh"

namespace mpk {

struct PendM { double v; unsigned long long key; unsigned idx, pad; };

// ring entry: the staged FP64 best (global key value) lands in (thr, pad) and fixup()
// replaces it in place by the FP32 filter threshold
struct alignas(16) E64 { double df, dg, a; float thr; unsigned pad; };

template <int DL, int G> struct Smem64f {
    using Gm = Geo<G, 1>;
    static constexpr int D = DL * G;
    static constexpr size_t ring_bytes =
        (((size_t)D * (Gm::PSR + Gm::PSC) * sizeof(E64)) + 15) & ~(size_t)15;
    // pending write-through merges (key slot, value, index), flushed by all lanes at once
    static constexpr int QN = 64;
    static constexpr size_t bytes_per_warp = ring_bytes + QN * sizeof(PendM);
    static constexpr int WPB = bytes_per_warp * 4 <= 112 * 1024 ? 4 : bytes_per_warp * 2 <= 112 * 1024 ? 2 : 1;
};

__device__ __forceinline__ float sqrt_abs_f(float x) {
    float r;
    asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(fabsf(x)));
    return r;
}

template <int DL, int G, bool SELF>
__global__ void __launch_bounds__(128)
mp_diag64f(const MainParams p) {
    using Gm = Geo<G, 1>;
    using SM = Smem64f<DL, G>;
    using KO = KeyOps<double>;
    using K = K64;
    constexpr int CA = Gm::CA, RA = Gm::RA, CW = Gm::CW, D = DL * G;
    constexpr int PSR = Gm::PSR, PSC = Gm::PSC, SB = Gm::SB;

    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned char* wbase = smem_raw + (size_t)warp * SM::bytes_per_warp;
    PendM* pend = reinterpret_cast<PendM*>(wbase + SM::ring_bytes);
    int npend = 0;  // warp-uniform
    E64* rowv = reinterpret_cast<E64*>(wbase);
    E64* colv = rowv + (size_t)D * PSR;

    const double4* __restrict__ st_q = reinterpret_cast<const double4*>(p.st_q);
    const double4* __restrict__ st_r = reinterpret_cast<const double4*>(p.st_r);
    const double* __restrict__ tw_q = reinterpret_cast<const double*>(p.tw_q);
    const double* __restrict__ tw_r = reinterpret_cast<const double*>(p.tw_r);
    const double* __restrict__ mu_q = reinterpret_cast<const double*>(p.mu_q);
    const double* __restrict__ mu_r = reinterpret_cast<const double*>(p.mu_r);
    K* keys = reinterpret_cast<K*>(p.keys);

    const long long n = p.n;
    const int d = p.d, m = p.m, H = p.H, HT = p.HT;
    const int n32 = (int)n;
    const double two_m = (double)(2 * m);
    const double INF = PT<double>::inf();
    // filter margin: relative FP32 rounding of S_k (D^2 -> float, approx sqrt, k adds)
    const double margin = 1.0 + ldexp(1.0, -20) + (double)d * ldexp(1.0, -22);

    const int lc = lane >> Gm::LOG_G, g = lane & (G - 1);
    const int a = lc >> Gm::LOG_CA, c = lc & (CA - 1);
    unsigned gmask_row = 0, gmask_col = 0;
#pragma unroll
    for (int cc = 0; cc < CA; ++cc) gmask_row |= 1u << (((a * CA + cc) << Gm::LOG_G) + g);
#pragma unroll
    for (int aa = 0; aa < RA; ++aa) gmask_col |= 1u << (((aa * CA + c) << Gm::LOG_G) + g);

    auto stage = [&](bool is_row, int base, int p_lo, int p_hi) {
        const int cnt = p_hi - p_lo;
        if (cnt <= 0) return;
        E64* buf = is_row ? rowv : colv;
        const int ps = is_row ? PSR : PSC;
        const double4* __restrict__ st = is_row ? st_q : st_r;
        const bool want_thr = is_row || SELF;
        for (int e = lane; e < cnt * D; e += 32) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            if (pos < 0 || pos >= n32) continue;
            const int sl = is_row ? Gm::srow(pos) : Gm::scol(pos);
            E64* dst = &buf[pl * ps + sl];
            if (pl < d) {
                const double4* src = st + (size_t)pos * d + pl;
                cp_async16(dst, src);
                cp_async8(&dst->a, &src->z);
            } else {  // padded dimension: a = +inf with QT = -1 gives D = +inf
                dst->df = 0; dst->dg = 0; dst->a = INF;
            }
            const int rk = rank_of_plane<DL, G>(pl);
            if (rk < d && want_thr) cp_async8(&dst->thr, &keys[(size_t)pos * d + rk].v);
            else *reinterpret_cast<double*>(&dst->thr) = -INF;  // never hit
        }
    };
    // FP32 filter thresholds from the landed FP64 bests (rounded up, widened by the margin)
    auto fixup = [&](bool is_row, int base, int p_lo, int p_hi) {
        const int cnt = p_hi - p_lo;
        if (cnt <= 0) return;
        E64* buf = is_row ? rowv : colv;
        const int ps = is_row ? PSR : PSC;
        for (int e = lane; e < cnt * D; e += 32) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            if (pos < 0 || pos >= n32) continue;
            const int sl = is_row ? Gm::srow(pos) : Gm::scol(pos);
            E64& en = buf[pl * ps + sl];
            en.thr = __double2float_ru(*reinterpret_cast<const double*>(&en.thr) * margin);
        }
    };
    // merge the pending (value, index) pairs into the global keys: one CAS loop per lane, so
    // the L2 round trips of a batch overlap instead of serialising behind single leaders
    auto flush = [&]() {
        __syncwarp();
        for (int q = lane; q < npend; q += 32) KO::merge(keys + pend[q].key, pend[q].v, pend[q].idx);
        npend = 0;
        __syncwarp();
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

        const long long delta = delta0 + (long long)a * CW + c;
        long long lo = max(r0, max(0ll, -delta));
        long long hi = min(r1, n - max(delta, 0ll));
        if (delta > p.delta_hi) hi = lo;
        const int dlt = (int)delta, lo32 = (int)lo, hi32 = (int)hi;

        double QT[DL];
        auto seed_cell = [&](long long row) {  // direct centred dot product, compensated
            double mq[DL], mr[DL], cmp[DL];
            const long long i0 = row, j0 = row + delta;
            load_dims<double, DL, G>(mu_q + i0 * D, g, mq);
            load_dims<double, DL, G>(mu_r + j0 * D, g, mr);
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) { QT[kk] = 0.0; cmp[kk] = 0.0; }
#pragma unroll 2
            for (int tt = 0; tt < m; ++tt) {
                double xq[DL], xr[DL];
                load_dims<double, DL, G>(tw_q + (i0 + tt) * D, g, xq);
                load_dims<double, DL, G>(tw_r + (j0 + tt) * D, g, xr);
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    const double y = (xq[kk] - mq[kk]) * (xr[kk] - mr[kk]) - cmp[kk];
                    const double t2 = QT[kk] + y;
                    cmp[kk] = (t2 - QT[kk]) - y;
                    QT[kk] = t2;
                }
            }
#pragma unroll
            for (int kk = 0; kk < DL; ++kk)
                if ((kk * G + g) >= d) QT[kk] = -1.0;
        };
#pragma unroll
        for (int kk = 0; kk < DL; ++kk) QT[kk] = (kk * G + g) >= d ? -1.0 : 0.0;
        int seeded_step = -1;

        const int nrows = (int)(r1 - r0);
        const int s_end = nrows + CW * (RA - 1);
        const int R0 = (int)r0, C0 = (int)(r0 + delta0);
        int row_in = min(SB, nrows), col_in = min(SB, s_end) + CW - 1;
        int fx_r0 = 0, fx_c0 = 0;
        stage(true, R0, 0, row_in);
        stage(false, C0, 0, col_in);
        cp_async_commit();
        cp_async_wait_all();
        __syncwarp();
        fixup(true, R0, 0, row_in);
        fixup(false, C0, 0, col_in);
        fx_r0 = row_in;
        fx_c0 = col_in;
        __syncwarp();

        auto step = [&](int s) {
            const int row = R0 + s - CW * a;
            const int col = row + dlt;
            const int sr = Gm::srow(row), sc = Gm::scol(col);
            const bool active = row >= lo32 && row < hi32;
            const bool upd = row > lo32 && row < hi32 && s != seeded_step;
            // ---- filter path: FP64 recurrence + D^2, FP32 distance / sort / scan / compare
            float Sf[DL], trf[DL], tcf[DL];
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) {
                const int pl = kk * G + g;
                const E64 R = rowv[pl * PSR + sr];
                const E64 C = colv[pl * PSC + sc];
                if (upd) QT[kk] = fma(R.df, C.dg, fma(C.df, R.dg, QT[kk]));      // Eq. (1)
                const double d2 = fma(-QT[kk], R.a * C.a, two_m);
                Sf[kk] = sqrt_abs_f(__double2float_rn(d2));
                trf[kk] = R.thr;
                tcf[kk] = C.thr;
            }
            sort_net<float, DL>(Sf);
            if (G > 1) lane_merge<float, DL, G>(Sf, g);
#pragma unroll
            for (int kk = 1; kk < DL; ++kk) Sf[kk] += Sf[kk - 1];
            if (G > 1) {
                float tot = Sf[DL - 1];
#pragma unroll
                for (int dd = 1; dd < G; dd <<= 1) {
                    const float y = __shfl_up_sync(FULL, tot, dd, G);
                    if (g >= dd) tot += y;
                }
                float excl = __shfl_up_sync(FULL, tot, 1, G);
                if (g == 0) excl = 0.f;
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) Sf[kk] += excl;
            }
            bool h[4] = {false, false, false, false};
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) {
                h[kk & 3] |= Sf[kk] <= trf[kk];
                if (SELF) h[kk & 3] |= Sf[kk] <= tcf[kk];
            }
            const bool hit = ((h[0] | h[1]) | (h[2] | h[3])) && active;
            if (!__any_sync(FULL, hit)) return;
            // ---- exact FP64 path for this warp step (Eqs. 1-3 in FP64)
            double S[DL];
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) {
                const int pl = kk * G + g;
                const double ra = rowv[pl * PSR + sr].a, ca = colv[pl * PSC + sc].a;
                S[kk] = PT<double>::sqrt_abs(fma(-QT[kk], ra * ca, two_m));
            }
            sort_net<double, DL>(S);
            if (G > 1) lane_merge<double, DL, G>(S, g);
#pragma unroll
            for (int kk = 1; kk < DL; ++kk) S[kk] += S[kk - 1];
            if (G > 1) {
                double tot = S[DL - 1];
#pragma unroll
                for (int dd = 1; dd < G; dd <<= 1) {
                    const double y = __shfl_up_sync(FULL, tot, dd, G);
                    if (g >= dd) tot += y;
                }
                double excl = __shfl_up_sync(FULL, tot, 1, G);
                if (g == 0) excl = 0.0;
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) S[kk] += excl;
            }
            if (!active) {
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) S[kk] = INF;
            }
            // ranks some lane can improve (one warp OR; the staged thresholds only decrease, so
            // this is a superset): the loop below skips the others without any vote
            unsigned rk_bits = 0;
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) {
                const int pl = kk * G + g;
                bool hk = S[kk] <= (double)rowv[pl * PSR + sr].thr;
                if (SELF) hk |= S[kk] <= (double)colv[pl * PSC + sc].thr;
                rk_bits |= (unsigned)hk << kk;
            }
            rk_bits = __reduce_or_sync(FULL, rk_bits);
            // Eq. (3), write-through: rank by rank (S rotates through S[0], so no dynamic
            // register indexing), group min by shuffles, the lowest-index leader merges
            // (value, index) into the global key and lowers the ring threshold
#pragma unroll 1
            for (int kk = 0; kk < DL; ++kk) {
                const int pl = kk * G + g;
                const double v = S[0];
#pragma unroll
                for (int q = 0; q + 1 < DL; ++q) S[q] = S[q + 1];
                if (((rk_bits >> kk) & 1u) == 0u) continue;
                const int rk = rank_of_plane<DL, G>(pl);
                const bool need_r = __any_sync(FULL, v <= (double)rowv[pl * PSR + sr].thr);
                const bool need_c = SELF && __any_sync(FULL, v <= (double)colv[pl * PSC + sc].thr);
                if (!need_r && !need_c) continue;
                double vr = v;
#pragma unroll
                for (int bit = 0; bit < Gm::LOG_CA; ++bit)
                    vr = PT<double>::vmin(vr, __shfl_xor_sync(FULL, vr, 1 << (bit + Gm::LOG_G)));
                const unsigned eqr = __ballot_sync(FULL, v == vr) & gmask_row;
                if (npend > SM::QN - 32) flush();  // room for one round of leaders (<= 32)
                const bool lead_r = need_r && vr < INF && rk < d && lane == __ffs(eqr) - 1;
                const unsigned lr = __ballot_sync(FULL, lead_r);
                if (lead_r) {
                    PendM& e = pend[npend + __popc(lr & ((1u << lane) - 1))];
                    e.v = vr;
                    e.key = (unsigned long long)row * d + rk;
                    e.idx = (unsigned)col;
                    float& th = rowv[pl * PSR + sr].thr;
                    th = fminf(th, __double2float_ru(vr * margin));
                }
                npend += __popc(lr);
                if (SELF && need_c) {
                    double vc = v;
#pragma unroll
                    for (int bit = 0; bit < 5 - Gm::LOG_G - Gm::LOG_CA; ++bit)
                        vc = PT<double>::vmin(vc, __shfl_xor_sync(FULL, vc, 1 << (bit + Gm::LOG_G + Gm::LOG_CA)));
                    const unsigned eqc = __ballot_sync(FULL, v == vc) & gmask_col;
                    if (npend > SM::QN - 32) flush();
                    const bool lead_c = vc < INF && rk < d && eqc != 0 && lane == 31 - __clz(eqc);
                    const unsigned lcm = __ballot_sync(FULL, lead_c);
                    if (lead_c) {
                        PendM& e = pend[npend + __popc(lcm & ((1u << lane) - 1))];
                        e.v = vc;
                        e.key = (unsigned long long)col * d + rk;
                        e.idx = (unsigned)row;
                        float& th = colv[pl * PSC + sc].thr;
                        th = fminf(th, __double2float_ru(vc * margin));
                    }
                    npend += __popc(lcm);
                }
            }
            __syncwarp();
        };

        int to_seed = SB;  // steps until the next seed (H is a multiple of SB)
        for (int s0 = 0; s0 < s_end; s0 += SB) {
            if ((to_seed -= SB) == 0) {  // seeds: first row at s0 = 0, current row every H steps
                to_seed = H;
                const long long row = R0 + s0 - (long long)CW * a;
                if (s0 == 0) { if (lo < hi) seed_cell(lo); }
                else if (row > lo && row < hi) seed_cell(row);
                seeded_step = s0 == 0 ? -1 : s0;
            }
            const int nxt = min(s0 + 2 * SB, s_end);
            const int r_need = min(nxt, nrows), c_need = nxt + CW - 1;
            stage(true, R0, row_in, r_need);
            stage(false, C0, col_in, c_need);
            row_in = max(row_in, r_need);
            col_in = max(col_in, c_need);
            cp_async_commit();
            const int s1 = min(s0 + SB, s_end);
#pragma unroll 1
            for (int ss = s0; ss < s1; ++ss) step(ss);
            if (npend) flush();
            cp_async_wait_all();
            __syncwarp();
            fixup(true, R0, fx_r0, row_in);
            fixup(false, C0, fx_c0, col_in);
            fx_r0 = row_in;
            fx_c0 = col_in;
            __syncwarp();
        }
        __syncwarp();
    }
}

template <int DL, int G, bool SELF> struct Inst64F {
    static size_t smem() { return Smem64f<DL, G>::bytes_per_warp * Smem64f<DL, G>::WPB; }
    static int warps_per_block() { return Smem64f<DL, G>::WPB; }
    static cudaError_t launch(const MainParams& p, int grid, cudaStream_t s);
    static int blocks_per_sm();
};

#ifdef MP_DIAG_IMPL
template <int DL, int G, bool SELF>
cudaError_t Inst64F<DL, G, SELF>::launch(const MainParams& p, int grid, cudaStream_t s) {
    const size_t sm = smem();
    cudaError_t e = cudaFuncSetAttribute(mp_diag64f<DL, G, SELF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    mp_diag64f<DL, G, SELF><<<grid, Smem64f<DL, G>::WPB * 32, sm, s>>>(p);
    return cudaGetLastError();
}
template <int DL, int G, bool SELF> int Inst64F<DL, G, SELF>::blocks_per_sm() {
    const size_t sm = smem();
    cudaFuncSetAttribute(mp_diag64f<DL, G, SELF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    int nb = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, mp_diag64f<DL, G, SELF>, Smem64f<DL, G>::WPB * 32, sm);
    return nb;
}
#endif

}  // namespace mpk

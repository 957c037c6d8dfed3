#pragma once
// mp_diag_cta64.cuh -- FP64 fused diagonal kernel for large d: the block-cooperative tiles of
// mp_diag_cta.cuh with the FP64-arithmetic + FP32-filter scheme of mp_diag64f.cuh.
//
// Method per cell (unchanged, Fig. 1: FP64 precalculation and main loop): QT
// recurrence and D^2 = 2m - QT a_i a_j in FP64 (Eq. 1); the sorted prefix sums
// (Eq. 2) are first formed in FP32 from D^2 rounded to FP32 and compared with FP32
// thresholds rounded UP and widened by a margin that bounds the FP32 rounding of S_k, so no
// cell that could improve a profile entry is filtered out.  A warp step where some lane passes
// re-runs the exact FP64 distance / sort / scan for its cells; each lane then merges every
// rank that beats the (hint) threshold into the global FP64 merge key with a 128-bit CAS
// (lexicographic (value, index) min, reading G2) -- Eq. 3, identical to a pure FP64 evaluation.
//
// Staging (why this kernel exists): an FP64 ring entry is 32 B per (position, dim), so at
// d >= 64 a warp-private ring held only 2-8 cells per warp and 3-6 warps per SM.  Here the NW
// warps of a block step through one tile together: the block's NT/G cells are consecutive
// diagonals in the SAME row, so per step the block stages one row and one column position
// into rings shared by all its warps.  Row updates (all cells of a step share the row) merge
// into a shared-memory FP64 key ring (128-bit CAS) that reaches the global key once per
// (row, rank) when the row leaves the ring (d <= 256; d = 512 writes through, the ring does
// not fit); column updates write through to the global key.  The
// FP32 filter thresholds in the ring are hints that only ever sit at or above the true
// (widened) best: a racing store can only leave one higher, which costs an extra exact pass,
// never a missed update.  Thresholds enter the ring as the key's FP64 value (cp.async into the
// entry's threshold word pair); after its own copies land each thread converts the entries it
// staged, then one block barrier per batch publishes them.
#include "mp_diag64f.cuh"

#ifndef MP_CTA64_ON
#define MP_CTA64_ON 1       // 0 switches the block-cooperative FP64 kernel off
#endif
#ifndef MP_CTA64_DL
#define MP_CTA64_DL 16      // dims per lane (G = d_pad / DL lanes per cell)
#endif
#ifndef MP_CTA64_MIN_DP
#define MP_CTA64_MIN_DP 64  // smallest padded d that takes it
#endif

namespace mpk {

// launch shape per lane-group size: warps per block, steps per staging batch
#ifndef MP_CTA64_SB
#define MP_CTA64_SB 0   // 0: per G below
#endif
// measured (n = 32768 / 8192 self-joins): d = 256 SB = 2 148 ms vs SB = 1 154 ms; d = 64 equal;
// d = 512 keeps SB = 1 (the rings fill the SM)
#ifndef MP_CTA64_NW_SMALLG
#define MP_CTA64_NW_SMALLG 4   // warps per block for d <= 128
#endif
#ifndef MP_CTA64_QN
#define MP_CTA64_QN 256   // per-block queue of global write-through merges, flushed once per batch (0: off)
#endif
#ifndef MP_CTA64_TA
#define MP_CTA64_TA 1   // FP32 filter thresholds in rank-contiguous per-slot arrays, read as vectors after the
                        // scan (none live through the sort: -32 registers), instead of the entries' thr word
#endif
#ifndef MP_CTA64_ROWKEY
#define MP_CTA64_ROWKEY 1   // row bests in a shared-memory key ring (d <= 256), merged at eviction
#endif
template <int G> struct CtaShape64 {
    static constexpr int NW = G >= 16 ? 8 : MP_CTA64_NW_SMALLG;
    // row key ring: the rows of a block tile are shared by all its cells, so their merges go
    // to shared memory (128-bit CAS) and reach the global key once per (row, rank) per tile;
    // it does not fit next to the d = 512 rings
    static constexpr bool ROWKEY = MP_CTA64_ROWKEY && G <= 16;
    static constexpr int SB = MP_CTA64_SB > 0 && G <= 16 ? MP_CTA64_SB : ((G == 16 && !ROWKEY) ? 2 : 1);
};

struct alignas(16) PendQ { unsigned long long key; double v; unsigned idx, pad0, pad1, pad2; };

// lexicographic (value, index) min into a shared-memory FP64 key (128-bit CAS)
__device__ __forceinline__ void smem_merge64(K64* p, double v, unsigned i) {
    const unsigned long long nv = (unsigned long long)__double_as_longlong(v), ni = i;
    const unsigned sa = (unsigned)__cvta_generic_to_shared(p);
    ulonglong2 old;
    asm volatile("ld.volatile.shared.v2.u64 {%0, %1}, [%2];" : "=l"(old.x), "=l"(old.y) : "r"(sa) : "memory");
    while (nv < old.x || (nv == old.x && ni < old.y)) {
        unsigned long long ox, oy;
        asm volatile(
            "{\n .reg .b128 c, n, o;\n mov.b128 c, {%2, %3};\n mov.b128 n, {%4, %5};\n"
            " atom.shared.cas.b128 o, [%6], c, n;\n mov.b128 {%0, %1}, o;\n}\n"
            : "=l"(ox), "=l"(oy)
            : "l"(old.x), "l"(old.y), "l"(nv), "l"(ni), "r"(sa)
            : "memory");
        if (ox == old.x && oy == old.y) break;
        old.x = ox;
        old.y = oy;
    }
}

template <int DL, int G, int NW> struct CtaGeo64 {
    static constexpr int NT = 32 * NW;   // threads per block
    static constexpr int NCC = NT / G;   // cells (diagonals) per block tile
    static constexpr int D = DL * G;
    static constexpr int SB = CtaShape64<G>::SB;
    // current batch + prefetch never share a slot (write-through: no eviction to wait for)
    static constexpr int RR = 3 * SB;
    static constexpr int RC = 3 * SB + NCC - 1;
    static constexpr bool ROWKEY = CtaShape64<G>::ROWKEY;
    static constexpr size_t base_bytes = (size_t)(RR + RC) * D * sizeof(E64) + (ROWKEY ? (size_t)RR * D * sizeof(K64) + 16 * ((RR * 4 + 15) / 16) : 0) + (size_t)MP_CTA64_QN * sizeof(PendQ) + 32;
    // threshold arrays where they fit next to the rings (not at d = 512)
    static constexpr bool TA = MP_CTA64_TA && base_bytes + (size_t)(RR + RC) * D * 4 <= 227 * 1024;
    static constexpr size_t ta_bytes = TA ? (size_t)(RR + RC) * D * 4 : 0;   // [slot][rank] float
    static constexpr size_t bytes = base_bytes + ta_bytes;
};

template <int DL, int G, int NW, bool SELF>
__global__ void __launch_bounds__(32 * NW, (NW == 4 ? 2 : 1))
mp_diag_cta64(const MainParams p) {
    using Cg = CtaGeo64<DL, G, NW>;
    using KO = KeyOps<double>;
    using K = K64;
    constexpr int D = Cg::D, NCC = Cg::NCC, RR = Cg::RR, RC = Cg::RC, SB = Cg::SB, NT = Cg::NT;

    extern __shared__ __align__(16) unsigned char smem_raw[];
    constexpr bool ROWKEY = Cg::ROWKEY;
    constexpr bool TA = Cg::TA;
    E64* rowv = reinterpret_cast<E64*>(smem_raw);
    E64* colv = rowv + (size_t)RR * D;
    K64* rowk = reinterpret_cast<K64*>(colv + (size_t)RC * D);                      // ROWKEY: [RR][D]
    unsigned* rdirty = reinterpret_cast<unsigned*>(rowk + (ROWKEY ? (size_t)RR * D : 0));
    constexpr int QN = MP_CTA64_QN;
    PendQ* pq = reinterpret_cast<PendQ*>(reinterpret_cast<unsigned char*>(rdirty) + (ROWKEY ? 16 * ((RR * 4 + 15) / 16) : 0));
    long long* tile_sh = reinterpret_cast<long long*>(pq + QN);
    unsigned* qn = reinterpret_cast<unsigned*>(tile_sh + 1);   // queued merges (monotone)
    float* ta = reinterpret_cast<float*>(tile_sh + 4);           // MP_CTA64_TA: thresholds [slot][rank], rows then columns

    const double4* __restrict__ st_q = reinterpret_cast<const double4*>(p.st_q);
    const double4* __restrict__ st_r = reinterpret_cast<const double4*>(p.st_r);
    const double* __restrict__ tw_q = reinterpret_cast<const double*>(p.tw_q);
    const double* __restrict__ tw_r = reinterpret_cast<const double*>(p.tw_r);
    const double* __restrict__ mu_q = reinterpret_cast<const double*>(p.mu_q);
    const double* __restrict__ mu_r = reinterpret_cast<const double*>(p.mu_r);
    K* keys = reinterpret_cast<K*>(p.keys);

    const long long n = p.n;
    const int n32 = (int)n;
    const int d = p.d, m = p.m, H = p.H, HT = p.HT;
    const double two_m = (double)(2 * m);
    const double INF = PT<double>::inf();
    // filter margin: relative FP32 rounding of S_k (D^2 -> float, approx sqrt, k adds)
    const double margin = 1.0 + ldexp(1.0, -20) + (double)d * ldexp(1.0, -22);
    const int tid = threadIdx.x;
    const int c = tid / G, g = tid & (G - 1);  // cell of the block tile, lane within the cell
    if (tid == 0) *qn = 0u;
    unsigned qbase = 0;                                         // block-uniform: flushed so far
    // global write-through merge, queued when there is room (the queue is flushed by all threads
    // at the batch end, so the L2 round trips of the CAS loops overlap instead of serialising
    // behind the lanes that hit)
    auto merge_q = [&](size_t key, double v, unsigned idx) {
        if constexpr (QN > 0) {
            const unsigned slot = atomicAdd(qn, 1u);
            if (slot - qbase < (unsigned)QN) {
                PendQ& e = pq[slot % QN];
                e.key = key; e.v = v; e.idx = idx;
                return;
            }
        }
        KO::merge(keys + key, v, idx);
    };

    const int off_r = ((n32 + RR) / RR) * RR, off_c = ((n32 + RC) / RC) * RC;
    auto rslot = [&](int pos) { return (pos + off_r) % RR; };
    auto cslot = [&](int pos) { return (pos + off_c) % RC; };

    // stage positions [p_lo, p_hi) of one side: (df, dg, a) and the FP64 best (into the
    // threshold word pair) by cp.async
    auto stage = [&](bool is_row, int base, int p_lo, int p_hi) {
        E64* buf = is_row ? rowv : colv;
        const double4* __restrict__ st = is_row ? st_q : st_r;
        const bool want_thr = is_row || SELF;
        const int cnt = p_hi - p_lo;
        for (int e = tid; e < cnt * D; e += NT) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            E64* dst = &buf[(is_row ? rslot(pos) : cslot(pos)) * D + pl];
            const int rk = rank_of_plane<DL, G>(pl);
            if (pos >= 0 && pos < n32 && pl < d) {
                const double4* src = st + (size_t)pos * d + pl;
                cp_async16(dst, src);
                cp_async8(&dst->a, &src->z);
            } else {  // padded dimension / past the end: a = +inf with QT = -1 gives D = +inf
                dst->df = 0; dst->dg = 0; dst->a = INF;
            }
            if (pos >= 0 && pos < n32 && rk < d && want_thr) cp_async8(&dst->thr, &keys[(size_t)pos * d + rk].v);
            else *reinterpret_cast<double*>(&dst->thr) = -INF;  // never hit
            if (ROWKEY && is_row) {
                const int sl = rslot(pos);
                if (pl == 0) rdirty[sl] = 0;
                K64* kd = &rowk[sl * D + pl];
                if (pos >= 0 && pos < n32 && rk < d) cp_async16(kd, &keys[(size_t)pos * d + rk]);
                else { kd->v = EMPTY64V; kd->i = EMPTY64I; }
            }
        }
    };
    // ROWKEY: merge the dirty row keys of positions [p_lo, p_hi) into the global keys
    auto evict_rows = [&](int base, int p_lo, int p_hi) {
        const int cnt = p_hi - p_lo;
        for (int e = tid; e < cnt * D; e += NT) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            if (pos < 0 || pos >= n32) continue;
            const int sl = rslot(pos);
            if (rdirty[sl] == 0) continue;
            const int rk = rank_of_plane<DL, G>(pl);
            if (rk >= d) continue;
            const K64 kv = rowk[sl * D + pl];
            if (kv.v < EMPTY64V) KO::merge(keys + (size_t)pos * d + rk, __longlong_as_double((long long)kv.v), (unsigned)kv.i);
        }
    };
    // after this thread's copies landed: FP32 filter thresholds (rounded up, widened)
    auto fixup = [&](bool is_row, int base, int p_lo, int p_hi) {
        E64* buf = is_row ? rowv : colv;
        const int cnt = p_hi - p_lo;
        for (int e = tid; e < cnt * D; e += NT) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            const int sl = is_row ? rslot(pos) : cslot(pos);
            E64& en = buf[sl * D + pl];
            const float t = __double2float_ru(*reinterpret_cast<const double*>(&en.thr) * margin);
            if (TA) ta[(is_row ? sl : RR + sl) * D + rank_of_plane<DL, G>(pl)] = t;
            else en.thr = t;
        }
    };

    for (;;) {
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

        const long long delta = delta0 + c;
        long long lo = max(r0, max(0ll, -delta));
        long long hi = min(r1, n - max(delta, 0ll));
        if (delta > p.delta_hi) hi = lo;
        const int lo32 = (int)lo, hi32 = (int)hi, dlt = (int)delta;

        double QT[DL];
        auto seed_cell = [&](long long row) {  // direct centred dot product, compensated
            constexpr int SC = (DL % 4 == 0) ? 4 : DL;
            const long long i0 = row, j0 = row + delta;
#pragma unroll
            for (int c0 = 0; c0 < DL; c0 += SC) {
                double mq[SC], mr[SC], cmp[SC], acc[SC];
                load_dims<double, SC, G>(mu_q + i0 * D + c0 * G, g, mq);
                load_dims<double, SC, G>(mu_r + j0 * D + c0 * G, g, mr);
#pragma unroll
                for (int kk = 0; kk < SC; ++kk) { acc[kk] = 0.0; cmp[kk] = 0.0; }
#pragma unroll 2
                for (int tt = 0; tt < m; ++tt) {
                    double xq[SC], xr[SC];
                    load_dims<double, SC, G>(tw_q + (i0 + tt) * D + c0 * G, g, xq);
                    load_dims<double, SC, G>(tw_r + (j0 + tt) * D + c0 * G, g, xr);
#pragma unroll
                    for (int kk = 0; kk < SC; ++kk) {
                        const double y = (xq[kk] - mq[kk]) * (xr[kk] - mr[kk]) - cmp[kk];
                        const double t2 = acc[kk] + y;
                        cmp[kk] = (t2 - acc[kk]) - y;
                        acc[kk] = t2;
                    }
                }
#pragma unroll
                for (int kk = 0; kk < SC; ++kk) QT[c0 + kk] = ((c0 + kk) * G + g) >= d ? -1.0 : acc[kk];
            }
        };
        if (lo < hi) {
            seed_cell(lo);
        } else {
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) QT[kk] = (kk * G + g) >= d ? -1.0 : 0.0;
        }

        const int nrows = (int)(r1 - r0);
        const int R0 = (int)r0, C0 = (int)(r0 + delta0);
        int row_in = min(SB, nrows), col_in = min(SB, nrows) + NCC - 1;
        stage(true, R0, 0, row_in);
        stage(false, C0, 0, col_in);
        cp_async_commit();
        cp_async_wait_all();
        fixup(true, R0, 0, row_in);
        fixup(false, C0, 0, col_in);
        __syncthreads();

        int seeded_step = -1;
        int to_seed = H;
        for (int s0 = 0; s0 < nrows; s0 += SB) {
            if (s0 > 0 && (to_seed -= SB) == 0) {
                to_seed = H;
                const long long row = R0 + s0;
                if (row > lo && row < hi) seed_cell(row);
                seeded_step = s0;
            }
            if (ROWKEY && s0 > 0) evict_rows(R0, s0 - SB, s0);  // the previous batch's rows
            const int nxt = min(s0 + 2 * SB, nrows);
            const int r_lo = row_in, c_lo = col_in;
            stage(true, R0, row_in, nxt);
            stage(false, C0, col_in, nxt + NCC - 1);
            row_in = max(row_in, nxt);
            col_in = max(col_in, nxt + NCC - 1);
            cp_async_commit();
            const int s1 = min(s0 + SB, nrows);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                const int row = R0 + s, col = row + dlt;
                const bool active = row >= lo32 && row < hi32;
                const bool upd = row > lo32 && row < hi32 && s != seeded_step;
                const int sr = rslot(row), sc = cslot(col);
                // ---- filter path: FP64 recurrence + D^2, FP32 distance / sort / scan / compare
                float Sf[DL];
                bool h[4] = {false, false, false, false};
                float* TRs = ta + (size_t)sr * D + g * DL;          // this lane's ranks g DL ..
                float* TCs = ta + (size_t)(RR + sc) * D + g * DL;
                {
                    [[maybe_unused]] float trf[TA ? 1 : DL], tcf[TA ? 1 : DL];
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) {
                        const int pl = kk * G + g;
                        const E64 R = rowv[sr * D + pl];
                        const E64 C = colv[sc * D + pl];
                        if (upd) QT[kk] = fma(R.df, C.dg, fma(C.df, R.dg, QT[kk]));      // Eq. (1)
                        const double d2 = fma(-QT[kk], R.a * C.a, two_m);
                        Sf[kk] = sqrt_abs_f(__double2float_rn(d2));
                        if constexpr (!TA) { trf[kk] = R.thr; tcf[kk] = C.thr; }
                    }
                    sort_net<float, DL>(Sf);
                    lane_merge<float, DL, G>(Sf, g);
#pragma unroll
                    for (int kk = 1; kk < DL; ++kk) Sf[kk] += Sf[kk - 1];
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
#pragma unroll
                    for (int kk = 0; kk < DL; kk += 4) {
                        if constexpr (TA) {
                            const float4 tr = *reinterpret_cast<const float4*>(TRs + kk);
                            h[0] |= Sf[kk] <= tr.x; h[1] |= Sf[kk + 1] <= tr.y; h[2] |= Sf[kk + 2] <= tr.z; h[3] |= Sf[kk + 3] <= tr.w;
                            if (SELF) {
                                const float4 tc = *reinterpret_cast<const float4*>(TCs + kk);
                                h[0] |= Sf[kk] <= tc.x; h[1] |= Sf[kk + 1] <= tc.y; h[2] |= Sf[kk + 2] <= tc.z; h[3] |= Sf[kk + 3] <= tc.w;
                            }
                        } else {
#pragma unroll
                            for (int q4 = 0; q4 < 4; ++q4) {
                                h[q4] |= Sf[kk + q4] <= trf[kk + q4];
                                if (SELF) h[q4] |= Sf[kk + q4] <= tcf[kk + q4];
                            }
                        }
                    }
                }
                const bool hit = ((h[0] | h[1]) | (h[2] | h[3])) && active;
                if (!__any_sync(FULL, hit)) continue;
                // ---- exact FP64 path for this warp step (Eqs. 1-3 in FP64)
                double S[DL];
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    const int pl = kk * G + g;
                    S[kk] = PT<double>::sqrt_abs(fma(-QT[kk], rowv[sr * D + pl].a * colv[sc * D + pl].a, two_m));
                }
                sort_net<double, DL>(S);
                lane_merge<double, DL, G>(S, g);
#pragma unroll
                for (int kk = 1; kk < DL; ++kk) S[kk] += S[kk - 1];
                {
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
                if (!active) continue;
                // Eq. (3), lane-local write-through: rank by rank (S rotates through S[0], no
                // dynamic register indexing), merge into the global key, lower the hint
#pragma unroll 1
                for (int kk = 0; kk < DL; ++kk) {
                    const int pl = kk * G + g;
                    const double v = S[0];
#pragma unroll
                    for (int qq = 0; qq + 1 < DL; ++qq) S[qq] = S[qq + 1];
                    const int rk = rank_of_plane<DL, G>(pl);
                    if (rk >= d) continue;
                    float& thr_r = TA ? TRs[kk] : rowv[sr * D + pl].thr;
                    if (v <= (double)thr_r) {
                        if constexpr (ROWKEY) {
                            smem_merge64(&rowk[sr * D + pl], v, (unsigned)col);
                            rdirty[sr] = 1;
                        } else {
                            merge_q((size_t)row * d + rk, v, (unsigned)col);
                        }
                        atomicMin(reinterpret_cast<unsigned*>(&thr_r), __float_as_uint(__double2float_ru(v * margin)));
                    }
                    if (SELF) {
                        float& thr_c = TA ? TCs[kk] : colv[sc * D + pl].thr;
                        if (v <= (double)thr_c) {
                            merge_q((size_t)col * d + rk, v, (unsigned)row);
                            atomicMin(reinterpret_cast<unsigned*>(&thr_c), __float_as_uint(__double2float_ru(v * margin)));
                        }
                    }
                }
            }
            cp_async_wait_all();               // this thread's prefetch landed ...
            fixup(true, R0, r_lo, row_in);     // ... so it converts the thresholds it staged
            fixup(false, C0, c_lo, col_in);
            __syncthreads();                   // publish; this batch's reads are all done
            if constexpr (QN > 0) {            // flush the queued merges with every thread
                const unsigned qnow = *reinterpret_cast<volatile unsigned*>(qn);
                if (qnow != qbase) {
                    const unsigned qend = min(qnow, qbase + (unsigned)QN);
                    for (unsigned j = qbase + tid; j < qend; j += NT) {
                        const PendQ e = pq[j % QN];
                        KO::merge(keys + e.key, e.v, e.idx);
                    }
                    qbase = qnow;
                    __syncthreads();           // queue slots free again
                }
            }
        }
        if (ROWKEY && nrows > 0) evict_rows(R0, ((nrows - 1) / SB) * SB, row_in);  // the last rows
    }
}

template <int DL, int G, int NW, bool SELF> struct InstCta64 {
    static size_t smem() { return CtaGeo64<DL, G, NW>::bytes; }
    static cudaError_t launch(const MainParams& p, int grid, cudaStream_t s);
    static int blocks_per_sm();
};

#ifdef MP_DIAG_IMPL
template <int DL, int G, int NW, bool SELF>
cudaError_t InstCta64<DL, G, NW, SELF>::launch(const MainParams& p, int grid, cudaStream_t s) {
    const size_t sm = smem();
    cudaError_t e = cudaFuncSetAttribute(mp_diag_cta64<DL, G, NW, SELF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    mp_diag_cta64<DL, G, NW, SELF><<<grid, 32 * NW, sm, s>>>(p);
    return cudaGetLastError();
}
template <int DL, int G, int NW, bool SELF> int InstCta64<DL, G, NW, SELF>::blocks_per_sm() {
    const size_t sm = smem();
    cudaFuncSetAttribute(mp_diag_cta64<DL, G, NW, SELF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    int nb = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, mp_diag_cta64<DL, G, NW, SELF>, 32 * NW, sm);
    return nb;
}
#endif

}  // namespace mpk

#pragma once
// mp_diag_cta.cuh -- FP32 fused diagonal kernel for large d (G >= 4 lanes per cell):
// block-cooperative tiles with block-shared staging rings.
//
// Same method and arithmetic as mp_diag (mp_diag.cuh): for every cell of a tile, the QT
// recurrence (Eq. 1), the distance (Eq. 1), the d-way sort
// (in-lane Batcher network + warp-shuffle bitonic merge across the G lanes of a cell) and the
// inclusive scan (Eq. 2), and the filtered min / argmin into the row and column
// profile (Eq. 3; self-join symmetry, reading G13).
//
// What changes for large d is the staging.  A position's statistics occupy d x 24 bytes of
// ring, and a warp-private ring needs ~3-5 positions per cell when a warp holds only 32/G
// cells -- for d = 256 that left 4 warps (8 cells) per SM.  Here the NW warps of a block step
// through one tile TOGETHER: the block's NT/G cells are consecutive diagonals in the SAME
// row (row = r0 + s), so the block stages one row position and one column position per step
// into rings shared by all its warps (~1.1 positions per cell), synchronising once per batch
// of SB steps.  Profile updates are lane-local: a lane whose prefix sum beats the staged
// threshold merges its (value, index) key into the ring entry with a shared-memory 64-bit
// atomicMin (lexicographic (value, index) min, reading G2) -- no cross-lane group reduction;
// dirty positions are merged into the global keys with one atomicMin per (rank, position)
// when they leave the ring.
#include "mp_diag.cuh"

#ifndef MP_CTA_SB
#define MP_CTA_SB 0   // steps per staging batch (one block barrier per batch); 0: per G below
#endif
#ifndef MP_CTA_MIN_DP
#define MP_CTA_MIN_DP 64   // smallest padded d that takes the block-cooperative kernel
#endif
#ifndef MP_CTA_NW
#define MP_CTA_NW 4   // warps per block of the block-cooperative large-d FP32 kernel (0: off)
#endif

namespace mpk {

template <int DL, int G, int NW> struct CtaGeo {
    static constexpr int NT = 32 * NW;             // threads per block
    static constexpr int NCC = NT / G;             // cells (diagonals) per block tile
    static constexpr int D = DL * G;
    // steps per staging batch (measured, d = 64 / 256: SB = 2 98 / 70 ms, SB = 1 102 / 54 ms)
    static constexpr int SB = MP_CTA_SB > 0 ? MP_CTA_SB : (G == 4 ? 2 : 1);
    // ring slots: positions of the current batch, the prefetched next one and the batch being
    // evicted stay distinct, so eviction reads and prefetch writes never touch the same slot
    static constexpr int RR = 3 * SB;
    static constexpr int RC = 3 * SB + NCC - 1;
    static constexpr int SS = D + G;               // V4 slot stride: consecutive slots shift banks
    static constexpr size_t bytes =
        ((size_t)(RR + RC) * SS * 16 + (size_t)(RR + RC) * D * 8 + (size_t)(RR + RC + 1) * 4 + 8 + 15) & ~(size_t)15;
};

// resident blocks per SM the register budget is sized for (shared memory allows 3 blocks of
// 4 warps up to d = 128, 2 at d = 256)
#ifndef MP_CTA_MINB
#define MP_CTA_MINB 3
#endif
template <int DL, int G, int NW, bool SELF>
__global__ void __launch_bounds__(32 * NW, (G <= 8 ? MP_CTA_MINB : 2))
mp_diag_cta(const MainParams p) {
    using Cg = CtaGeo<DL, G, NW>;
    using V4 = float4;
    using K = unsigned long long;
    constexpr int D = Cg::D, NCC = Cg::NCC, RR = Cg::RR, RC = Cg::RC, SS = Cg::SS, SB = Cg::SB, NT = Cg::NT;
    constexpr int FOLD = SB > MP_FOLD ? SB : MP_FOLD;  // steps between folds of QL into QT

    extern __shared__ __align__(16) unsigned char smem_raw[];
    V4* rowv = reinterpret_cast<V4*>(smem_raw);
    V4* colv = rowv + (size_t)RR * SS;
    K* rowk = reinterpret_cast<K*>(colv + (size_t)RC * SS);
    K* colk = rowk + (size_t)RR * D;
    unsigned* rdirty = reinterpret_cast<unsigned*>(colk + (size_t)RC * D);
    unsigned* cdirty = rdirty + RR;
    long long* tile_sh = reinterpret_cast<long long*>(cdirty + RC + ((RR + RC) & 1));

    const V4* __restrict__ st_q = reinterpret_cast<const V4*>(p.st_q);
    const V4* __restrict__ st_r = reinterpret_cast<const V4*>(p.st_r);
    const float* __restrict__ tw_q = reinterpret_cast<const float*>(p.tw_q);
    const float* __restrict__ tw_r = reinterpret_cast<const float*>(p.tw_r);
    const float* __restrict__ mu_q = reinterpret_cast<const float*>(p.mu_q);
    const float* __restrict__ mu_r = reinterpret_cast<const float*>(p.mu_r);
    K* keys = reinterpret_cast<K*>(p.keys);

    const long long n = p.n;
    const int n32 = (int)n;
    const int d = p.d, m = p.m, H = p.H, HT = p.HT;
    const float two_m = (float)(2 * m);
    const float NINF = __int_as_float(0xff800000);
    const int tid = threadIdx.x;
    const int c = tid / G, g = tid & (G - 1);  // cell of the block tile, lane within the cell

    // stage positions [p_lo, p_hi) (relative to base) of one side into its ring: stats
    // (df, dg, a) and the threshold (.w = value half of the merge key) by cp.async, the full
    // key into the key ring; slots are cleared of their dirty flag
    // ring slot of a position: (pos + off) mod slots, off a multiple of the slot count >= n so
    // that AB-join columns below 0 (never-hit padding) still map to valid slots
    const int off_r = ((n32 + RR - 1) / RR) * RR, off_c = ((n32 + RC - 1) / RC) * RC;
    auto stage = [&](bool is_row, int base, int p_lo, int p_hi) {
        V4* buf = is_row ? rowv : colv;
        K* kb = is_row ? rowk : colk;
        unsigned* df = is_row ? rdirty : cdirty;
        const int nslot = is_row ? RR : RC;
        const V4* __restrict__ st = is_row ? st_q : st_r;
        const bool want_thr = is_row || SELF;
        const int cnt = p_hi - p_lo;
        for (int e = tid; e < cnt * D; e += NT) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            const int sl = (pos + (is_row ? off_r : off_c)) % nslot;
            if (pl == 0) df[sl] = 0;
            V4* dst = &buf[sl * SS + pl];
            K* kd = &kb[sl * D + pl];
            const int rk = rank_of_plane<DL, G>(pl);
            if (pos >= 0 && pos < n32 && pl < d) {
                const V4* src = st + (size_t)pos * d + pl;
                cp_async8(dst, src);
                cp_async4(&dst->z, &src->z);
            } else {  // padded dimension / position past the end: D ~ 1e18 (sorts last), never hit
                dst->x = 0.f; dst->y = 0.f; dst->z = PT<float>::pad_a();
            }
            if (pos >= 0 && pos < n32 && rk < d && want_thr) {
                const K* ks = keys + (size_t)pos * d + rk;
                cp_async4(&dst->w, reinterpret_cast<const char*>(ks) + 4);
                cp_async8(kd, ks);
            } else {
                dst->w = NINF;
                *kd = EMPTY32;
            }
        }
    };
    // merge dirty ring keys of leaving positions into the global keys
    auto evict = [&](bool is_row, int base, int p_lo, int p_hi) {
        if (!is_row && !SELF) return;
        const K* kb = is_row ? rowk : colk;
        const unsigned* df = is_row ? rdirty : cdirty;
        const int nslot = is_row ? RR : RC;
        const int cnt = p_hi - p_lo;
        for (int e = tid; e < cnt * D; e += NT) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            if (pos < 0 || pos >= n32) continue;
            const int sl = (pos + (is_row ? off_r : off_c)) % nslot;
            if (df[sl] == 0) continue;
            const int rk = rank_of_plane<DL, G>(pl);
            if (rk >= d) continue;
            const K kv = kb[sl * D + pl];
            if (kv < EMPTY32) atomicMin(keys + (size_t)pos * d + rk, kv);
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

        // this thread's cell: diagonal delta, valid rows [lo, hi)
        const long long delta = delta0 + c;
        long long lo = max(r0, max(0ll, -delta));
        long long hi = min(r1, n - max(delta, 0ll));
        if (delta > p.delta_hi) hi = lo;
        const int lo32 = (int)lo, hi32 = (int)hi, dlt = (int)delta;

        // QT = QT[kk] + QL[kk] (compensated, reading R4; see mp_diag)
        float QT[DL], QL[DL];
        auto seed_cell = [&](long long row) {  // direct centred dot product, compensated
            constexpr int SC = (DL % MP_SEED_CHUNK == 0) ? MP_SEED_CHUNK : DL;
            const long long i0 = row, j0 = row + delta;
            const float* xq_p = tw_q + i0 * D;
            const float* xr_p = tw_r + j0 * D;
#pragma unroll
            for (int c0 = 0; c0 < DL; c0 += SC) {
                float mq[SC], mr[SC], cmp[SC], acc[SC];
                load_dims<float, SC, G>(mu_q + i0 * D + c0 * G, g, mq);
                load_dims<float, SC, G>(mu_r + j0 * D + c0 * G, g, mr);
#pragma unroll
                for (int kk = 0; kk < SC; ++kk) { acc[kk] = 0.f; cmp[kk] = 0.f; }
#pragma unroll 2
                for (int tt = 0; tt < m; ++tt) {
                    float xq[SC], xr[SC];
                    load_dims<float, SC, G>(xq_p + (long long)tt * D + c0 * G, g, xq);
                    load_dims<float, SC, G>(xr_p + (long long)tt * D + c0 * G, g, xr);
#pragma unroll
                    for (int kk = 0; kk < SC; ++kk) {
                        const float y = (xq[kk] - mq[kk]) * (xr[kk] - mr[kk]) - cmp[kk];
                        const float t2 = acc[kk] + y;
                        cmp[kk] = (t2 - acc[kk]) - y;
                        acc[kk] = t2;
                    }
                }
#pragma unroll
                for (int kk = 0; kk < SC; ++kk) {  // the Kahan sum is acc - cmp: keep both words
                    const bool pad = ((c0 + kk) * G + g) >= d;
                    QT[c0 + kk] = pad ? -1.f : acc[kk];
                    QL[c0 + kk] = pad ? 0.f : -cmp[kk];
                }
            }
        };
        if (lo < hi) {
            seed_cell(lo);
        } else {
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) { QT[kk] = (kk * G + g) >= d ? -1.f : 0.f; QL[kk] = 0.f; }
        }

        const int nrows = (int)(r1 - r0);
        const int R0 = (int)r0, C0 = (int)(r0 + delta0);  // row / first column of step 0
        int row_in = min(SB, nrows), col_in = min(SB, nrows) + NCC - 1;
        stage(true, R0, 0, row_in);
        stage(false, C0, 0, col_in);
        cp_async_commit();
        cp_async_wait_all();
        __syncthreads();

        int seeded_step = -1;
        int to_seed = H;
        for (int s0 = 0; s0 < nrows; s0 += SB) {
            if ((s0 & (FOLD - 1)) == 0) {  // fold the increments into QT (exact Fast2Sum)
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    const float t = QT[kk] + QL[kk];
                    QL[kk] = QL[kk] - (t - QT[kk]);
                    QT[kk] = t;
                }
            }
            if (s0 > 0 && (to_seed -= SB) == 0) {
                to_seed = H;
                const long long row = R0 + s0;
                if (row > lo && row < hi) seed_cell(row);
                seeded_step = s0;
            }
            // evict the previous batch (its slots are not the ones prefetched below)
            if (s0 > 0) {
                evict(true, R0, s0 - SB, s0);
                evict(false, C0, s0 - SB, s0);
            }
            const int nxt = min(s0 + 2 * SB, nrows);
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
                const int sr = (R0 + s + off_r) % RR;
                const int sc = (C0 + s + c + off_c) % RC;
                float S[DL];
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    const int pl = kk * G + g;
                    const V4 R = rowv[sr * SS + pl];
                    const V4 C = colv[sc * SS + pl];
                    if (upd) QL[kk] = fmaf(R.x, C.y, fmaf(C.x, R.y, QL[kk]));          // Eq. (1)
                    const float pr = R.z * C.z;
                    S[kk] = PT<float>::sqrt_abs(fmaf(-QL[kk], pr, fmaf(-QT[kk], pr, two_m)));  // Eq. (1)
                }
                sort_net<float, DL>(S);                                               // Eq. (2)
                if constexpr (MP_FUSE_LAST && G > 1) {
                    lane_merge<float, DL, G, true>(S, g);
                    pair_scan<float, DL>(S);                                          // Eq. (2) scan
                } else {
                    lane_merge<float, DL, G>(S, g);
#pragma unroll
                    for (int kk = 1; kk < DL; ++kk) S[kk] += S[kk - 1];                // Eq. (2) scan
                }
                {
                    float tot = S[DL - 1];
#pragma unroll
                    for (int dd = 1; dd < G; dd <<= 1) {
                        const float y = __shfl_up_sync(FULL, tot, dd, G);
                        if (g >= dd) tot += y;
                    }
                    float excl = __shfl_up_sync(FULL, tot, 1, G);
                    if (g == 0) excl = 0.f;
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) S[kk] += excl;
                }
                // Eq. (3): threshold test against the staged bests (plane kk*G+g holds the
                // threshold of rank g*DL+kk, the rank this lane holds at kk after the merge)
                bool h[4] = {false, false, false, false};
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    const int pl = kk * G + g;
                    h[kk & 3] |= S[kk] <= rowv[sr * SS + pl].w;
                    if (SELF) h[kk & 3] |= S[kk] <= colv[sc * SS + pl].w;
                }
                if (((h[0] | h[1]) | (h[2] | h[3])) && active) {
                    // lane-local update: 64-bit shared atomicMin on the ring key (value bits
                    // << 32 | index: lexicographic, lowest index on ties), lower the threshold
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) {
                        const int pl = kk * G + g;
                        const float v = S[kk];
                        const unsigned vb = __float_as_uint(v);
                        if (v <= rowv[sr * SS + pl].w) {
                            atomicMin(&rowk[sr * D + pl], ((K)vb << 32) | (unsigned)col);
                            atomicMin(reinterpret_cast<unsigned*>(&rowv[sr * SS + pl].w), vb);
                            rdirty[sr] = 1;
                        }
                        if (SELF && v <= colv[sc * SS + pl].w) {
                            atomicMin(&colk[sc * D + pl], ((K)vb << 32) | (unsigned)row);
                            atomicMin(reinterpret_cast<unsigned*>(&colv[sc * SS + pl].w), vb);
                            cdirty[sc] = 1;
                        }
                    }
                }
            }
            cp_async_wait_all();
            __syncthreads();  // prefetch landed for all threads; this batch's reads and updates done
        }
        // epilogue: evict everything still live (the last batch and the columns after it)
        if (nrows > 0) {
            const int s_last = ((nrows - 1) / SB) * SB;
            evict(true, R0, s_last, row_in);
            evict(false, C0, s_last, col_in);
        }
    }
}

template <int DL, int G, int NW, bool SELF> struct InstCta {
    static size_t smem() { return CtaGeo<DL, G, NW>::bytes; }
    static int warps_per_block() { return NW; }
    static cudaError_t launch(const MainParams& p, int grid, cudaStream_t s);
    static int blocks_per_sm();
};

#ifdef MP_DIAG_IMPL
template <int DL, int G, int NW, bool SELF>
cudaError_t InstCta<DL, G, NW, SELF>::launch(const MainParams& p, int grid, cudaStream_t s) {
    const size_t sm = smem();
    cudaError_t e = cudaFuncSetAttribute(mp_diag_cta<DL, G, NW, SELF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    mp_diag_cta<DL, G, NW, SELF><<<grid, 32 * NW, sm, s>>>(p);
    return cudaGetLastError();
}
template <int DL, int G, int NW, bool SELF> int InstCta<DL, G, NW, SELF>::blocks_per_sm() {
    const size_t sm = smem();
    cudaFuncSetAttribute(mp_diag_cta<DL, G, NW, SELF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    int nb = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, mp_diag_cta<DL, G, NW, SELF>, 32 * NW, sm);
    return nb;
}
#endif

}  // namespace mpk

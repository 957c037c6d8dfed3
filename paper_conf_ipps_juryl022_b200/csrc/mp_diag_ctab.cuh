#pragma once
// mp_diag_ctab.cuh -- FP32 fused diagonal kernel for large d (d >= 64): block-cooperative
// tiles, TMA bulk staging, 32 dims per lane.
//
// Method per cell (Fig. 1 FP32 main loop; reading R4): the compensated QT
// recurrence (Eq. 1), the distance (Eq. 1), the d-way sort and inclusive
// scan (Eq. 2) and the filtered min / argmin into the row and column profile
// (Eq. 3; self-join symmetry, reading G13).
//
// What this kernel does differently from the first block-cooperative kernel (mp_diag_cta):
//   * a lane holds DL = 32 dims of a cell (G = d_pad / 32 lanes per cell): the in-lane Batcher
//     network sorts 32 values and only log2(G) bitonic merge levels cross lanes (d = 64: one
//     level, 1 SHFL per cell*dim instead of 3);
//   * staging is Blackwell-native: each entering position's statistics (d x 16 B, contiguous
//     in the position-major stats array) arrive by ONE cp.async.bulk (TMA) issued by one thread,
//     completing on an mbarrier; the threshold words are patched in afterwards from the merge
//     keys (loaded one batch ahead into registers);
//   * profile updates write through: a lane whose prefix sum passes the staged threshold merges
//     its (value, index) key into the global key with a 64-bit RED.MIN (lexicographic
//     (value, index) min, reading G2) and lowers the ring's threshold hint with a shared 32-bit
//     atomicMin.  The hint is only ever >= the global best (it was read from the key, or
//     lowered to a value that was merged), so filtering with it never loses an update.  There
//     is no key ring and no eviction pass, which halves the shared memory per position;
//   * QT is compensated (QT + QL, reading R4): increments accumulate in QL, folded into QT by
//     an exact Fast2Sum every FOLD steps; the seeds keep both words of their Kahan sums.
#include "mp_diag.cuh"

#ifndef MP_CTAB_ON
#define MP_CTAB_ON 1        // 0: large-d FP32 takes mp_diag_cta (cp.async staging, DL = 16)
#endif
#ifndef MP_CTAB_NT
#define MP_CTAB_NT 128      // threads per block
#endif
#ifndef MP_CTAB_MINB16
#define MP_CTAB_MINB16 4    // resident blocks per SM the register budget is sized for (DL = 16: 127 registers, no spills)
#endif
#ifndef MP_CTAB_MINB32
#define MP_CTAB_MINB32 3    // ... (DL = 32)
#endif
#ifndef MP_CTAB_SB
#define MP_CTAB_SB 0        // steps per staging batch; 0: per G below
#endif
#ifndef MP_CTAB_PAIR
#define MP_CTAB_PAIR 1      // G == 2: the pair-mode merge (pair_si)
#endif
#ifndef MP_CTAB_SIGN
#define MP_CTAB_SIGN 0      // G == 4: sign-split cross-lane merge (two of three cross-lane steps uniform;
                            // measured C3 -1 % time but the negative lanes' prefix sums cancel: off)
#endif
#ifndef MP_CTAB_TA
#define MP_CTAB_TA 1        // thresholds in rank-contiguous per-slot arrays (read as vectors after
                            // the scan) instead of the stats' 4th word (kept live through the sort)
#endif
// dims per lane by padded d (G = d_pad / DL lanes per cell, G <= 32)
#ifndef MP_CTAB_DL64
#define MP_CTAB_DL64 16
#endif
#ifndef MP_CTAB_DL128
#define MP_CTAB_DL128 16
#endif
#ifndef MP_CTAB_DL256
#define MP_CTAB_DL256 16
#endif
#ifndef MP_CTAB_DL512
#define MP_CTAB_DL512 16
#endif

namespace mpk {

constexpr int ctab_dl(int dp) {
    return dp <= 64 ? MP_CTAB_DL64 : dp <= 128 ? MP_CTAB_DL128 : dp <= 256 ? MP_CTAB_DL256 : dp <= 512 ? MP_CTAB_DL512 : 32;
}

template <int DL, int G, int NT> struct CtabGeo {
    static constexpr int NCC = NT / G;                 // cells (diagonals) per block tile
    static constexpr int D = DL * G;                   // padded dims
    static constexpr int SB = MP_CTAB_SB > 0 ? MP_CTAB_SB : (NT / G >= 32 ? 2 : 1);
    // ring slots: the current batch and the prefetched one (no eviction pass: write-through)
    static constexpr int RR = 2 * SB;
    static constexpr int RC = 2 * SB + NCC - 1;
    static constexpr int SS = D + G;                   // V4 slot stride: consecutive slots shift banks
    static constexpr int NTHR = (2 * SB * D + NT - 1) / NT;  // threshold words a thread patches per batch
    static constexpr size_t stat_ring_bytes = (size_t)(RR + RC) * SS * 16;
    static constexpr size_t ring_bytes = stat_ring_bytes + (MP_CTAB_TA ? (size_t)(RR + RC) * D * 4 : 0);
    static constexpr size_t bytes = ring_bytes + 16 /* mbarrier */ + 16 /* tile index */;
};

// plane (dimension slot) that holds rank r's threshold: lane g holds ranks [g DL, (g+1) DL) at
// registers kk after the merge and reads plane kk G + g at register kk (rank_of_plane inverse)
template <int DL, int G> __device__ __forceinline__ int plane_of_rank(int r) { return (r % DL) * G + r / DL; }

// Pair mode (G == 2, MP_CTAB_PAIR): the upper lane of a cell negates its distances before the
// in-lane sort, so after the sort it holds its run negated and reversed.  The cross-lane bitonic
// "flip" then pairs equal register indices and is the same instruction in both lanes,
// s = min(s, -partner(s)): one SHFL + one FMNMX per element and no lane-dependent min / max (which
// costs FMNMX + predicated FMNMX), and the in-lane half-cleaners stay ascending in both lanes.
// Padded dims have D = 0 exactly (a = 1, QT = 2m) and sort FIRST: sorted index si = rank + npad.
// After the fused scan of the stored values P_g, lane 0 register j holds S at sorted index j;
// lane 1 register j <= DL - 2 holds sorted index 2 DL - 2 - j (= c_1 + P_1[j] with
// c_1 = P_0[DL - 1] - P_1[DL - 1]) and register DL - 1 the total (sorted index 2 DL - 1).
template <int DL> __device__ __forceinline__ int pair_si(int g, int kk) {
    return g == 0 ? kk : (kk == DL - 1 ? 2 * DL - 1 : 2 * DL - 2 - kk);
}
// position of sorted index si in the per-slot threshold array: lane g's registers are contiguous
template <int DL> __device__ __forceinline__ int pair_pos_of_si(int si) {
    return si < DL ? si : (si == 2 * DL - 1 ? 2 * DL - 1 : 3 * DL - 2 - si);
}

// Sign-split merge (G == 4, MP_CTAB_SIGN).  Lanes 2 and 3 of a cell hold their distances negated
// (stored value = sigma_g x true value, sigma = (+, +, -, -)).  A cross-lane compare between lanes of
// opposite sign is then the same instruction in both lanes, own = min(own, -partner): the positive
// lane keeps the true minimum, the negative lane the true maximum (negated) -- one FMNMX with a
// negated operand instead of a lane-dependent min / max pair (FMNMX + predicated FMNMX).  The
// 64-element merge of four sorted 16-runs: (1) lanes g ^ 2, same register: uniform; in-lane
// half-cleaners; (2) lanes g ^ 3, same register: uniform; (3) lanes g ^ 1, mirrored register
// (same-sign pairs: lane-dependent); in-lane half-cleaners (the last layer fused into pair_scan).
// Result (checked exhaustively against a sort in the stage self-test): lane 0 holds true ranks
// 0..15 ascending, lane 1 16..31, lane 2 ranks 47 - k at register k, lane 3 ranks 63 - k, all as
// stored values ascending.  Derived by searching the uniform-step sequences.
template <int DL> __device__ __forceinline__ void sign_merge4(float (&v)[DL], int g) {
    static_assert((DL & (DL - 1)) == 0 && DL >= 4, "power-of-two DL");
#pragma unroll
    for (int kk = 0; kk < DL; ++kk) v[kk] = fminf(v[kk], -__shfl_xor_sync(FULL, v[kk], 2));
#pragma unroll
    for (int dist = DL / 2; dist >= 1; dist >>= 1)
#pragma unroll
        for (int kk = 0; kk < DL; ++kk)
            if ((kk & dist) == 0) cswap(v[kk], v[kk + dist]);
#pragma unroll
    for (int kk = 0; kk < DL; ++kk) v[kk] = fminf(v[kk], -__shfl_xor_sync(FULL, v[kk], 3));
    const bool keep_min = g == 0 || g == 3;   // stored minimum: lanes 0 (+, true min) and 3 (-, true max)
#pragma unroll
    for (int kk = 0; kk < DL / 2; ++kk) {
        const float y1 = __shfl_xor_sync(FULL, v[DL - 1 - kk], 1);
        const float y2 = __shfl_xor_sync(FULL, v[kk], 1);
        v[kk] = keep_min ? fminf(v[kk], y1) : fmaxf(v[kk], y1);
        v[DL - 1 - kk] = keep_min ? fminf(v[DL - 1 - kk], y2) : fmaxf(v[DL - 1 - kk], y2);
    }
#pragma unroll
    for (int dist = DL / 2; dist >= 2; dist >>= 1)
#pragma unroll
        for (int kk = 0; kk < DL; ++kk)
            if ((kk & dist) == 0) cswap(v[kk], v[kk + dist]);
}
// true rank held at register kk of lane g after sign_merge4
template <int DL> __device__ __forceinline__ int sign_rank(int g, int kk) {
    return g < 2 ? g * DL + kk : (kk == DL - 1 ? (g + 1) * DL - 1 : (g + 1) * DL - 2 - kk);
}
// position of rank r in a lane-blocked threshold array read by register (sign_rank inverse)
template <int DL> __device__ __forceinline__ int sign_pos(int r) {
    const int b = r / DL, i = r - b * DL;
    return b < 2 ? r : b * DL + (i == DL - 1 ? DL - 1 : DL - 2 - i);
}
// after pair_scan of the stored values (inclusive prefix P_k in register k): the true prefix sums
// S at the ranks sign_rank(g, k).  t_g = sigma_g P_{DL-1} is the lane's true total; c_g = sum of
// the totals of the lanes holding lower ranks (positive lanes) or of lanes up to g (negative lanes,
// whose register k < DL - 1 then holds c_g + P_k = S at rank (g + 1) DL - 2 - k, and the last
// register the lane's end S = c_g).
template <int DL> __device__ __forceinline__ void sign_offsets(float (&v)[DL], int g) {
    const float pos = g < 2 ? 1.f : 0.f;
    const float t = (g < 2) ? v[DL - 1] : -v[DL - 1];
    float incl = t;
#pragma unroll
    for (int dd = 1; dd < 4; dd <<= 1) {
        const float y = __shfl_up_sync(FULL, incl, dd, 4);
        if (g >= dd) incl += y;
    }
    const float c = fmaf(-pos, t, incl);   // positive lanes: exclusive prefix; negative: inclusive
#pragma unroll
    for (int kk = 0; kk < DL - 1; ++kk) v[kk] += c;
    v[DL - 1] = fmaf(pos, v[DL - 1], c);
}

template <int DL, int G, int NT, bool SELF>
__global__ void __launch_bounds__(NT, DL <= 16 ? MP_CTAB_MINB16 : MP_CTAB_MINB32) mp_diag_ctab(const MainParams p) {
    using Cg = CtabGeo<DL, G, NT>;
    using V4 = float4;
    using K = unsigned long long;
    constexpr int D = Cg::D, NCC = Cg::NCC, RR = Cg::RR, RC = Cg::RC, SS = Cg::SS, SB = Cg::SB;
    constexpr int NTHR = Cg::NTHR;
    constexpr bool PM = MP_CTAB_PAIR && MP_CTAB_TA && G == 2;   // pair mode (pair_si)
    constexpr bool SM = MP_CTAB_SIGN && MP_CTAB_TA && G == 4;    // sign-split merge (sign_merge4)
    constexpr int FOLD = SB > MP_FOLD ? SB : MP_FOLD;

    extern __shared__ __align__(16) unsigned char smem_raw[];
    V4* rowv = reinterpret_cast<V4*>(smem_raw);
    V4* colv = rowv + (size_t)RR * SS;
    unsigned long long* bar = reinterpret_cast<unsigned long long*>(smem_raw + Cg::ring_bytes);
    long long* tile_sh = reinterpret_cast<long long*>(smem_raw + Cg::ring_bytes + 16);

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
    const unsigned stat_bytes = (unsigned)d * 16u;
    const int npad = D - d;
    // padded planes: pair mode D = 0 (a = 1, QT = 2m; sorts first), else D ~ 1e18 (sorts last)
    constexpr bool ZP = PM || SM;   // padded dims have D = 0 exactly (sort first; ranks shift by npad)
    const float pad_a = ZP ? 1.f : PT<float>::pad_a();

    // padded planes [d, D) never change (TMA writes planes [0, d) of a slot): set them once
    for (int e = tid; e < (RR + RC) * (D - d); e += NT) {
        const int sl = e / (D - d), pl = d + e % (D - d);
        V4* dst = (sl < RR ? rowv + (size_t)sl * SS : colv + (size_t)(sl - RR) * SS) + pl;
        *dst = make_float4(0.f, 0.f, pad_a, NINF);
    }
    if (tid == 0) {
        mbar_init(bar, 1);   // thread 0 arrives once per batch (issue_batch)
        fence_proxy_async();
    }
    unsigned phase = 0;
    const int off_r = ((n32 + RR - 1) / RR) * RR, off_c = ((n32 + RC - 1) / RC) * RC;
    auto rslot = [&](int pos) { return (pos + off_r) % RR; };
    auto cslot = [&](int pos) { return (pos + off_c) % RC; };

    // TMA staging of positions [p_lo, p_hi) of one side (relative to base): one bulk copy per
    // in-range position by thread 0; out-of-range positions (AB-join / band edges) are filled
    // by all threads as never-hit padding.  Returns nothing; thread 0 arms the mbarrier once per
    // batch with the total byte count (issue_batch).
    auto issue_batch = [&](int R0, int r_lo, int r_hi, int C0, int c_lo, int c_hi) {
        if (tid == 0) {
            unsigned bytes = 0;
            for (int q = r_lo; q < r_hi; ++q) bytes += stat_bytes;  // rows are always in range
            for (int q = c_lo; q < c_hi; ++q) {
                const int pos = C0 + q;
                if (pos >= 0 && pos < n32) bytes += stat_bytes;
            }
            mbar_arrive_expect_tx(bar, bytes);
            for (int q = r_lo; q < r_hi; ++q) {
                const int pos = R0 + q;
                bulk_g2s(rowv + (size_t)rslot(pos) * SS, st_q + (size_t)pos * d, stat_bytes, bar);
            }
            for (int q = c_lo; q < c_hi; ++q) {
                const int pos = C0 + q;
                if (pos >= 0 && pos < n32)
                    bulk_g2s(colv + (size_t)cslot(pos) * SS, st_r + (size_t)pos * d, stat_bytes, bar);
            }
        }
        for (int q = c_lo; q < c_hi; ++q) {  // out-of-range columns: padding (rare, warp-uniform test)
            const int pos = C0 + q;
            if (pos >= 0 && pos < n32) continue;
            V4* dst = colv + (size_t)cslot(pos) * SS;
            for (int pl = tid; pl < D; pl += NT) dst[pl] = make_float4(0.f, 0.f, pad_a, NINF);
        }
    };
    // threshold words of the staged positions: entry e = (position index, rank r); rank r's
    // threshold sits in plane plane_of_rank(r).  Rows: the query profile's key; columns
    // (self-join only): the key of the column position.
    // (dst: float index of the threshold word in the rings)
    float* const ringf = reinterpret_cast<float*>(smem_raw);
    auto thr_entry = [&](int e, int R0, int r_lo, int nr, int C0, int c_lo, int& dst) -> float {
        const int pi = e / D, q = e - pi * D;   // q: rank (pair mode: sorted index, rank q - npad)
        const bool is_row = pi < nr;
        const int pos = is_row ? R0 + r_lo + pi : C0 + c_lo + (pi - nr);
        const int slot = is_row ? rslot(pos) : RR + cslot(pos);
        if (MP_CTAB_TA) dst = (int)(Cg::stat_ring_bytes / 4) + slot * D + (PM ? pair_pos_of_si<DL>(q) : SM ? sign_pos<DL>(q) : q);
        else dst = (slot * SS + plane_of_rank<DL, G>(q)) * 4 + 3;
        const int r = ZP ? q - npad : q;
        if (r < 0 || r >= d || pos < 0 || pos >= n32) return NINF;
        return __uint_as_float(__ldcg(reinterpret_cast<const unsigned*>(keys + (size_t)pos * d + r) + 1));
    };

    for (;;) {
        fence_proxy_async();   // this thread's generic writes to the rings precede later TMA writes
        __syncthreads();       // previous tile fully done (rings, tile_sh)
        if (tid == 0) *tile_sh = (long long)atomicAdd(p.counter, 1ull);
        __syncthreads();
        const long long t = *tile_sh;
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

        const int nrows = (int)(r1 - r0);
        const int R0 = (int)r0, C0 = (int)(r0 + delta0);  // row / first column of step 0
        int row_in = min(SB, nrows), col_in = min(SB, nrows) + NCC - 1;
        issue_batch(R0, 0, row_in, C0, 0, col_in);   // overlaps the seeds below

        // QT = QT[kk] + QL[kk] (compensated, reading R4); seeds: direct centred dot products
        // (reading G8) with Kahan sums, both words kept.  The seed operands
        // are position-major with each lane's DL dims contiguous (pre_pm, PreParams::pm_G), so
        // they load as 16-byte vectors.
        float QT[DL], QL[DL];
        auto seed_cell = [&](long long row) {
            constexpr int SC = 4;
            const long long i0 = row, j0 = row + delta;
            const float* xq_p = tw_q + i0 * D + g * DL;
            const float* xr_p = tw_r + j0 * D + g * DL;
#pragma unroll
            for (int c0 = 0; c0 < DL; c0 += SC) {
                const float4 mq = __ldg(reinterpret_cast<const float4*>(mu_q + i0 * D + g * DL + c0));
                const float4 mr = __ldg(reinterpret_cast<const float4*>(mu_r + j0 * D + g * DL + c0));
                float acc[SC] = {0.f, 0.f, 0.f, 0.f}, cmp[SC] = {0.f, 0.f, 0.f, 0.f};
#pragma unroll 2
                for (int tt = 0; tt < m; ++tt) {
                    const float4 xq = __ldg(reinterpret_cast<const float4*>(xq_p + (long long)tt * D + c0));
                    const float4 xr = __ldg(reinterpret_cast<const float4*>(xr_p + (long long)tt * D + c0));
                    const float pq[SC] = {xq.x - mq.x, xq.y - mq.y, xq.z - mq.z, xq.w - mq.w};
                    const float pr[SC] = {xr.x - mr.x, xr.y - mr.y, xr.z - mr.z, xr.w - mr.w};
#pragma unroll
                    for (int kk = 0; kk < SC; ++kk) {
                        const float y = fmaf(pq[kk], pr[kk], -cmp[kk]);
                        const float t2 = acc[kk] + y;
                        cmp[kk] = (t2 - acc[kk]) - y;
                        acc[kk] = t2;
                    }
                }
#pragma unroll
                for (int kk = 0; kk < SC; ++kk) {  // lane g's register c0 + kk is dim (c0 + kk) G + g
                    const bool pad = ((c0 + kk) * G + g) >= d;
                    QT[c0 + kk] = pad ? (ZP ? two_m : -1.f) : acc[kk];
                    QL[c0 + kk] = pad ? 0.f : -cmp[kk];
                }
            }
        };
        if (lo < hi) {
            seed_cell(lo);
        } else {
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) { QT[kk] = (kk * G + g) >= d ? (ZP ? two_m : -1.f) : 0.f; QL[kk] = 0.f; }
        }

        // first batch landed: patch its thresholds directly (once per tile)
        mbar_wait(bar, phase);
        phase ^= 1;
        {
            const int nr = row_in, nc = SELF ? col_in : 0;
            for (int e = tid; e < (nr + nc) * D; e += NT) {
                int dst;
                const float v = thr_entry(e, R0, 0, nr, C0, 0, dst);
                ringf[dst] = v;
            }
        }
        __syncthreads();

        int seeded_step = -1;
        int to_seed = H;
        for (int s0 = 0; s0 < nrows; s0 += SB) {
            if ((s0 & (FOLD - 1)) == 0) {  // fold the increments into QT (exact Fast2Sum)
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    const float t2 = QT[kk] + QL[kk];
                    QL[kk] = QL[kk] - (t2 - QT[kk]);
                    QT[kk] = t2;
                }
            }
            if (s0 > 0 && (to_seed -= SB) == 0) {
                to_seed = H;
                const long long row = R0 + s0;
                if (row > lo && row < hi) seed_cell(row);
                seeded_step = s0;
            }
            // prefetch the next batch: stats by TMA, thresholds into registers
            const int nxt = min(s0 + 2 * SB, nrows);
            const int r_lo = row_in, r_hi = max(row_in, nxt);
            const int c_lo = col_in, c_hi = max(col_in, nxt + NCC - 1);
            issue_batch(R0, r_lo, r_hi, C0, c_lo, c_hi);
            const int nr = r_hi - r_lo, nc = SELF ? c_hi - c_lo : 0;
            float thv[NTHR];
            int thp[NTHR];
#pragma unroll
            for (int k = 0; k < NTHR; ++k) {
                const int e = tid + k * NT;
                thp[k] = -1;
                thv[k] = NINF;
                if (e < (nr + nc) * D) thv[k] = thr_entry(e, R0, r_lo, nr, C0, c_lo, thp[k]);
            }
            row_in = r_hi;
            col_in = c_hi;

            const int s1 = min(s0 + SB, nrows);
#pragma unroll 1
            for (int s = s0; s < s1; ++s) {
                const int row = R0 + s, col = row + dlt;
                const bool active = row >= lo32 && row < hi32;
                const bool upd = row > lo32 && row < hi32 && s != seeded_step;
                const int sr = rslot(row), sc = cslot(C0 + s + c);
                const V4* Rs = rowv + (size_t)sr * SS;
                const V4* Cs = colv + (size_t)sc * SS;
                // thresholds of this lane's ranks g DL .. g DL + DL - 1 (MP_CTAB_TA)
                float* TRs = ringf + Cg::stat_ring_bytes / 4 + (size_t)sr * D + g * DL;
                float* TCs = ringf + Cg::stat_ring_bytes / 4 + (size_t)(RR + sc) * D + g * DL;
                float S[DL];
                [[maybe_unused]] float thr[MP_CTAB_TA ? 1 : DL];
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    const int pl = kk * G + g;
                    const V4 R = Rs[pl];
                    const V4 C = Cs[pl];
                    if (upd) QL[kk] = fmaf(R.x, C.y, fmaf(C.x, R.y, QL[kk]));              // Eq. (1)
                    const float pr = R.z * C.z;
                    S[kk] = PT<float>::sqrt_abs(fmaf(-QL[kk], pr, fmaf(-QT[kk], pr, two_m)));  // Eq. (1)
                    // plane kk G + g carries the threshold of rank g DL + kk: the rank this
                    // lane holds at register kk after the sort (one test covers row and column)
                    if constexpr (!MP_CTAB_TA) thr[kk] = SELF ? fmaxf(R.w, C.w) : R.w;
                }
                if constexpr (SM) {
                    const float sgn = g < 2 ? 1.f : -1.f;
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) S[kk] *= sgn;
                }
                if constexpr (PM) {
                    const float sgn = g ? -1.f : 1.f;
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) S[kk] *= sgn;
                }
                sort_net<float, DL>(S);                                                  // Eq. (2)
                if constexpr (PM) {
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) S[kk] = fminf(S[kk], -__shfl_xor_sync(FULL, S[kk], 1));
#pragma unroll
                    for (int dist = DL / 2; dist >= 2; dist >>= 1)
#pragma unroll
                        for (int kk = 0; kk < DL; ++kk)
                            if ((kk & dist) == 0) cswap(S[kk], S[kk + dist]);
                    pair_scan<float, DL>(S);                                             // Eq. (2) scan
                    const float tot = S[DL - 1];
                    const float oth = __shfl_xor_sync(FULL, tot, 1);
                    const float cg = g ? oth - tot : 0.f;
#pragma unroll
                    for (int kk = 0; kk < DL - 1; ++kk) S[kk] += cg;
                    S[DL - 1] = g ? cg : tot;
                } else if constexpr (SM) {
                    sign_merge4<DL>(S, g);
                    pair_scan<float, DL>(S);                                             // Eq. (2) scan
                    sign_offsets<DL>(S, g);
                } else {
                if constexpr (G > 1) lane_merge<float, DL, G, true>(S, g);
                pair_scan<float, DL>(S);                                                 // Eq. (2) scan
                }
                if constexpr (G > 1 && !PM && !SM) {
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
                bool h[4] = {false, false, false, false};
#pragma unroll
                for (int kk = 0; kk < DL; kk += 4) {
                    if constexpr (MP_CTAB_TA) {
                        const float4 tr = *reinterpret_cast<const float4*>(TRs + kk);
                        h[0] |= S[kk] <= tr.x; h[1] |= S[kk + 1] <= tr.y; h[2] |= S[kk + 2] <= tr.z; h[3] |= S[kk + 3] <= tr.w;
                        if (SELF) {
                            const float4 tc = *reinterpret_cast<const float4*>(TCs + kk);
                            h[0] |= S[kk] <= tc.x; h[1] |= S[kk + 1] <= tc.y; h[2] |= S[kk + 2] <= tc.z; h[3] |= S[kk + 3] <= tc.w;
                        }
                    } else {
#pragma unroll
                        for (int q = 0; q < 4; ++q) h[q] |= S[kk + q] <= thr[kk + q];
                    }
                }
                if (((h[0] | h[1]) | (h[2] | h[3])) && active) {
                    // Eq. (3), write-through: merge into the global key, lower the hint
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) {
                        const float v = S[kk];
                        const int pl = kk * G + g, rk = PM ? pair_si<DL>(g, kk) - npad : SM ? sign_rank<DL>(g, kk) - npad : g * DL + kk;
                        const unsigned vb = __float_as_uint(v);
                        float* rw = MP_CTAB_TA ? TRs + kk : const_cast<float*>(&Rs[pl].w);
                        if (v <= *reinterpret_cast<volatile float*>(rw)) {
                            atomicMin(keys + (size_t)row * d + rk, ((K)vb << 32) | (unsigned)col);
                            atomicMin(reinterpret_cast<unsigned*>(rw), vb);
                        }
                        if (SELF) {
                            float* cw = MP_CTAB_TA ? TCs + kk : const_cast<float*>(&Cs[pl].w);
                            if (v <= *reinterpret_cast<volatile float*>(cw)) {
                                atomicMin(keys + (size_t)col * d + rk, ((K)vb << 32) | (unsigned)row);
                                atomicMin(reinterpret_cast<unsigned*>(cw), vb);
                            }
                        }
                    }
                }
            }
            mbar_wait(bar, phase);   // the next batch's statistics have landed
            phase ^= 1;
#pragma unroll
            for (int k = 0; k < NTHR; ++k)
                if (thp[k] >= 0) ringf[thp[k]] = thv[k];
            fence_proxy_async();
            __syncthreads();  // thresholds published; this batch's reads and updates done
        }
    }
}

template <int DL, int G, int NT, bool SELF> struct InstCtab {
    static_assert(G >= 2 && G <= 32 && DL * G >= 64, "block-cooperative FP32 kernel: 2..32 lanes per cell");
    static size_t smem() { return CtabGeo<DL, G, NT>::bytes; }
    static int warps_per_block() { return NT / 32; }
    static cudaError_t launch(const MainParams& p, int grid, cudaStream_t s);
    static int blocks_per_sm();
};

#ifdef MP_DIAG_IMPL
template <int DL, int G, int NT, bool SELF>
cudaError_t InstCtab<DL, G, NT, SELF>::launch(const MainParams& p, int grid, cudaStream_t s) {
    const size_t sm = smem();
    cudaError_t e = cudaFuncSetAttribute(mp_diag_ctab<DL, G, NT, SELF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    mp_diag_ctab<DL, G, NT, SELF><<<grid, NT, sm, s>>>(p);
    return cudaGetLastError();
}
template <int DL, int G, int NT, bool SELF> int InstCtab<DL, G, NT, SELF>::blocks_per_sm() {
    const size_t sm = smem();
    cudaFuncSetAttribute(mp_diag_ctab<DL, G, NT, SELF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    int nb = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, mp_diag_ctab<DL, G, NT, SELF>, NT, sm);
    return nb;
}
#endif

}  // namespace mpk

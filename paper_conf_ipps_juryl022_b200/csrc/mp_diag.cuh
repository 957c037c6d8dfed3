#pragma once
// mp_kernels.cu -- hand-written sm_100a kernels of the mSTAMP hot path.
//
// Paper: Ju et al., "Exploiting Reduced Precision for GPU-based Time Series Mining",
// IPDPS 2022 (/root/reference/PAPER.md, cited PAPER.md:L<n>).  DESIGN.md explains the
// design; this file implements:
//   * precompute  -- per-window mean / norm (two-pass), df, dg, a = sqrt(2m)/norm
//                    ("precalculation"; reading G7)
//   * mp_diag     -- the fused hot kernel: for every cell of a W-diagonal x H-row tile
//                    QT recurrence (Eq. 1) -> distance (Eq. 1) ->
//                    d-way sort + inclusive scan (Eq. 2) -> filtered
//                    min/argmin into the row AND column profile (Eq. 3,
//                    self-join symmetry, reading G13).  D, D', D'' never leave registers.
//   * finalize    -- merge keys -> P (mean = sum/(k+1)), I (reading G11).
//
// Execution model (B200-first, not the paper's 3-kernels-per-row loop):
//   one warp owns a tile of NC consecutive diagonals x H rows; G lanes cooperate on a
//   cell when d > 32 (each holds DL dims), and for small d a lane owns W = 2 adjacent
//   diagonals (same row, columns j and j+1; column j+1's data is carried in registers to
//   the next step, halving shared-memory traffic).  The lane-cells of a warp step are
//   arranged as RA rows x CA columns (row = r0 + s - CA*W*a) so a step touches RA rows
//   and CA*W columns.  Row/column statistics and the running profile thresholds are
//   staged in per-warp shared-memory rings by cp.async (LDGSTS) one step ahead.  The
//   profile update is filtered: a cell only does work if some S_k <= current best of
//   its row or column (fresh per warp, seeded from global memory at row entry); such
//   steps run a warp-shuffle group-min + leader update, and dirty rows/columns are
//   merged into global memory with one 64-bit (FP32) / 128-bit CAS (FP64) atomic per
//   (rank, position) when they leave the ring.  Persistent warps pull tiles from an
//   atomic counter.
#include <cuda_runtime.h>
#include <cstdint>
#include <cmath>
#include "mp_internal.h"
#ifndef MP_MINB
#define MP_MINB 1
#endif
#ifndef MP_MINB_F32
#define MP_MINB_F32 3
#endif
#ifndef MP_W1_UNROLL
#define MP_W1_UNROLL 1
#endif
#define MP_PRAGMA(x) _Pragma(#x)
#define MP_UNROLL(n) MP_PRAGMA(unroll n)
#ifndef MP_CA_W2
#define MP_CA_W2 4   // lanes per row group for two cells per lane (half kernel d <= 16, FP32 d <= 8)
#endif
#ifndef MP_FUSE_LAST
#define MP_FUSE_LAST 1   // fuse the final sort / merge layer into the scan (C2 FP32 40.35 -> 39.8 ms)
#endif
#ifndef MP_SLOW_UNROLL
#define MP_SLOW_UNROLL 0   // 1: slow path over register-resident S, unrolled over the ranks (spills: C2 FP32 39.6 -> 48.9 ms)
#endif
#ifndef MP_KEEP_DL
#define MP_KEEP_DL 16
#endif
#ifndef MP_FOLD
#define MP_FOLD 4   // steps between the Fast2Sum folds of the compensated QT (power of two)
#endif
#ifndef MP_SEED_CHUNK
#define MP_SEED_CHUNK 4
#endif
// steps per staging batch by lanes-per-cell G: wide cells (large d) keep fewer positions in
// flight so the per-warp rings stay small enough for several resident warps per SM
#ifndef MP_SB_G1
#define MP_SB_G1 4
#endif
#ifndef MP_SB_G2
#define MP_SB_G2 2
#endif
#ifndef MP_SB_G4
#define MP_SB_G4 1
#endif

namespace mpk {

constexpr unsigned FULL = 0xffffffffu;
constexpr int WARPS_PER_BLOCK = 4;
constexpr unsigned DIRTY = 0x80000000u;
constexpr unsigned EMPTY_IDX = 0x7FFFFFFFu;   // ring index of a slot without a local find

// ------------------------------------------------------------------ precision traits
template <class T> struct PT;
template <> struct PT<float> {
    using V4 = float4;
    // 'a' of padded dimensions / positions: D = sqrt(|2m - QT a a|) ~ 1e18 sorts last; finite,
    // so the compensated evaluation fma(-QT_lo, a a, .) never forms 0 * inf
    static __device__ __forceinline__ float pad_a() { return 1e18f; }
    static __device__ __forceinline__ float inf() { return __int_as_float(0x7f800000); }
    static __device__ __forceinline__ float ninf() { return __int_as_float(0xff800000); }
    // sqrt of |x|: |x| absorbs the rounding residue of 2m - QT a_i a_j near D = 0
    // (reading G5); MUFU.SQRT with the free |.| modifier.  Relative error ~2^-22, far
    // below the FP32 tolerance.
    static __device__ __forceinline__ float sqrt_abs(float x) {
        float r;
        asm("sqrt.approx.ftz.f32 %0, %1;" : "=f"(r) : "f"(fabsf(x)));
        return r;
    }
    static __device__ __forceinline__ float vmin(float a, float b) { return fminf(a, b); }
    static __device__ __forceinline__ float vmax(float a, float b) { return fmaxf(a, b); }
};
template <> struct PT<double> {
    using V4 = double4;
    static __device__ __forceinline__ double pad_a() { return 1e18; }
    static __device__ __forceinline__ double inf() { return __longlong_as_double(0x7ff0000000000000ll); }
    static __device__ __forceinline__ double ninf() { return __longlong_as_double((long long)0xfff0000000000000ull); }
    static __device__ __forceinline__ double sqrt_abs(double x) { return sqrt(fabs(x)); }  // IEEE RN
    static __device__ __forceinline__ double vmin(double a, double b) { return b < a ? b : a; }
    static __device__ __forceinline__ double vmax(double a, double b) { return b < a ? a : b; }
};

template <class T> __device__ __forceinline__ void cswap(T& a, T& b) {
    T lo = PT<T>::vmin(a, b), hi = PT<T>::vmax(a, b);
    a = lo;
    b = hi;
}

// Ampere-style async global->shared copies (LDGSTS): ring staging without registers.
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(sa), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async8(void* smem, const void* gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 8;\n" ::"r"(sa), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async4(void* smem, const void* gmem) {
    const unsigned sa = (unsigned)__cvta_generic_to_shared(smem);
    asm volatile("cp.async.ca.shared.global [%0], [%1], 4;\n" ::"r"(sa), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
__device__ __forceinline__ void cp_async_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }

// ------------------------------------------------------------------ TMA / mbarrier helpers
__device__ __forceinline__ unsigned smem_u32(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(unsigned long long* bar, unsigned bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
                 : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(unsigned long long* bar, unsigned parity) {
    unsigned ok;
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    return ok != 0;
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned parity) {
    while (!mbar_try_wait(bar, parity)) {
    }
}
// one bulk global -> shared copy (16-byte aligned, size a multiple of 16) completing on bar
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, unsigned long long* bar) {
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(dst)),
                 "l"(src), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
// order this thread's generic-proxy shared-memory accesses before later async-proxy (TMA) ones
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// Batcher odd-even merge sort network on N registers (any N), ascending (Eq. 2 "sort",
// PAPER.md:L642-643, reading G12).  The comparator list is generated at compile time
// (constexpr) so every register index is a constant after unrolling.
constexpr int batcher_count(int N) {
    int c = 0;
    for (int p = 1; p < N; p <<= 1)
        for (int k = p; k >= 1; k >>= 1)
            for (int j = k % p; j + k < N; j += 2 * k)
                for (int i = 0; i < k; ++i)
                    if (i + j + k < N && (i + j) / (2 * p) == (i + j + k) / (2 * p)) ++c;
    return c;
}
template <int N> struct BatcherNet {
    static constexpr int C = batcher_count(N) > 0 ? batcher_count(N) : 1;
    short a[C], b[C];
    constexpr BatcherNet() : a{}, b{} {
        int c = 0;
        for (int p = 1; p < N; p <<= 1)
            for (int k = p; k >= 1; k >>= 1)
                for (int j = k % p; j + k < N; j += 2 * k)
                    for (int i = 0; i < k; ++i)
                        if (i + j + k < N && (i + j) / (2 * p) == (i + j + k) / (2 * p)) {
                            a[c] = (short)(i + j);
                            b[c] = (short)(i + j + k);
                            ++c;
                        }
    }
};
template <class T, int N> __device__ __forceinline__ void sort_net(T (&v)[N]) {
    if constexpr (N > 1) {
        constexpr BatcherNet<N> net{};
#pragma unroll
        for (int c = 0; c < batcher_count(N); ++c) cswap(v[net.a[c]], v[net.b[c]]);
    }
}

// All comparators of sort_net but the final layer's N/2 - 1 adjacent ones (i, i+1), i odd
// (for a power of two N the generator emits that layer last).  The caller fuses that layer
// into the inclusive scan: S_i = S_{i-1} + min(v_i, v_{i+1}), S_{i+1} = S_{i-1} + (v_i + v_{i+1})
// -- the larger value is never formed, which moves N/2 - 1 min/max ops from the ALU pipe to
// FADDs on the FMA pipe and halves the scan's dependency chain.
template <int N> constexpr bool last_layer_adjacent() {
    if (N < 4 || (N & (N - 1))) return false;
    const BatcherNet<N> net{};
    for (int t = 0; t < N / 2 - 1; ++t) {
        const int c = batcher_count(N) - 1 - t;
        if (net.a[c] != N - 3 - 2 * t || net.b[c] != N - 2 - 2 * t) return false;
    }
    return true;
}
template <class T, int N> __device__ __forceinline__ void sort_net_head(T (&v)[N]) {
    static_assert(last_layer_adjacent<N>(), "final Batcher layer must be the adjacent odd pairs");
    constexpr BatcherNet<N> net{};
#pragma unroll
    for (int c = 0; c < batcher_count(N) - (N / 2 - 1); ++c) cswap(v[net.a[c]], v[net.b[c]]);
}
// sort_net_head + the fused final layer + inclusive scan: v becomes S_0..S_{N-1}
template <class T, int N> __device__ __forceinline__ void sort_scan_fused(T (&v)[N]) {
    sort_net_head<T, N>(v);
    T lo[N / 2], pr[N / 2];  // lo[h], pr[h]: min and sum of the pair (2h-1, 2h), h >= 1
#pragma unroll
    for (int h = 1; h < N / 2; ++h) {
        lo[h] = PT<T>::vmin(v[2 * h - 1], v[2 * h]);
        pr[h] = v[2 * h - 1] + v[2 * h];
    }
    // even prefix chain E_h = S_{2h} (two half chains joined), then the odd entries
    T E[N / 2];
    E[0] = v[0];
    constexpr int HH = N / 4;  // second chain starts at h = HH
#pragma unroll
    for (int h = 1; h < HH; ++h) E[h] = E[h - 1] + pr[h];
    T F = pr[HH];
#pragma unroll
    for (int h = HH + 1; h < N / 2; ++h) { E[h] = F + pr[h]; F = E[h]; }
#pragma unroll
    for (int h = HH; h < N / 2; ++h) E[h] = (h == HH ? pr[h] : E[h]) + E[HH - 1];
    const T last = v[N - 1];
#pragma unroll
    for (int h = 1; h < N / 2; ++h) v[2 * h - 1] = E[h - 1] + lo[h];
#pragma unroll
    for (int h = 0; h < N / 2; ++h) v[2 * h] = E[h];
    v[N - 1] = E[N / 2 - 1] + last;
}

// In-lane inclusive scan fused with a final layer of adjacent pairs (2h, 2h+1) left out by
// lane_merge<..., true>: S_{2h} = E_{h-1} + min, S_{2h+1} = E_{h-1} + (v_{2h} + v_{2h+1}).
template <class T, int DL> __device__ __forceinline__ void pair_scan(T (&v)[DL]) {
    static_assert(DL >= 4 && (DL & (DL - 1)) == 0, "pair_scan needs a power-of-two DL >= 4");
    constexpr int NH = DL / 2, HH = NH / 2;
    T lo[NH], E[NH];
#pragma unroll
    for (int h = 0; h < NH; ++h) {
        lo[h] = PT<T>::vmin(v[2 * h], v[2 * h + 1]);
        E[h] = v[2 * h] + v[2 * h + 1];
    }
    // prefix over the pair sums in two half chains joined at the end
#pragma unroll
    for (int h = 1; h < HH; ++h) E[h] = E[h] + E[h - 1];
#pragma unroll
    for (int h = HH + 1; h < NH; ++h) E[h] = E[h] + E[h - 1];
#pragma unroll
    for (int h = HH; h < NH; ++h) E[h] = E[h] + E[HH - 1];
    v[0] = lo[0];
    v[1] = E[0];
#pragma unroll
    for (int h = 1; h < NH; ++h) {
        v[2 * h] = E[h - 1] + lo[h];
        v[2 * h + 1] = E[h];
    }
}

// Bitonic merge of the sorted DL-blocks held by G consecutive lanes (lane-blocked order:
// lane g ends up with ranks [g*DL, (g+1)*DL)).  The paper's group-cooperative bitonic
// sort expressed with warp shuffles instead of shared memory.
// SKIP_LAST: leave out the final in-lane stage (adjacent pairs (2h, 2h+1)) for pair_scan
template <class T, int DL, int G, bool SKIP_LAST = false>
__device__ __forceinline__ void lane_merge(T (&v)[DL], int g) {
#pragma unroll
    for (int p = 1; p < G; p <<= 1) {
        const bool lower = (g & p) == 0;
        // flip step: element kk of this lane vs element DL-1-kk of the mirrored lane
#pragma unroll
        for (int kk = 0; kk < DL / 2; ++kk) {
            T y1 = __shfl_xor_sync(FULL, v[DL - 1 - kk], 2 * p - 1);
            T y2 = __shfl_xor_sync(FULL, v[kk], 2 * p - 1);
            v[kk] = lower ? PT<T>::vmin(v[kk], y1) : PT<T>::vmax(v[kk], y1);
            v[DL - 1 - kk] = lower ? PT<T>::vmin(v[DL - 1 - kk], y2) : PT<T>::vmax(v[DL - 1 - kk], y2);
        }
        if (DL == 1) {  // (DL/2 == 0) degenerate block
            T y = __shfl_xor_sync(FULL, v[0], 2 * p - 1);
            v[0] = lower ? PT<T>::vmin(v[0], y) : PT<T>::vmax(v[0], y);
        }
        // half-cleaners across lanes
#pragma unroll
        for (int q = p >> 1; q >= 1; q >>= 1) {
            const bool lo = (g & q) == 0;
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) {
                T y = __shfl_xor_sync(FULL, v[kk], q);
                v[kk] = lo ? PT<T>::vmin(v[kk], y) : PT<T>::vmax(v[kk], y);
            }
        }
        // half-cleaners inside the lane
#pragma unroll
        for (int dist = DL / 2; dist >= ((SKIP_LAST && 2 * p == G) ? 2 : 1); dist >>= 1) {
#pragma unroll
            for (int kk = 0; kk < DL; ++kk)
                if ((kk & dist) == 0) cswap(v[kk], v[kk + dist]);
        }
    }
}

// ------------------------------------------------------------------ merge keys
// FP32: key = (float bits of S << 32) | j   (non-negative floats are order-isomorphic
//       to their bits, so u64 min == lexicographic (value, index) min, reading G2).
// FP64: {double bits of S, j} compared lexicographically, merged by 128-bit CAS.
// Empty entries carry index 0x7FFFFFFF so a staged index never has the DIRTY bit.
constexpr unsigned long long EMPTY32 = 0x7F8000007FFFFFFFull;          // (+inf, 2^31-1)
constexpr unsigned long long EMPTY64V = 0x7FF0000000000000ull;         // +inf
constexpr unsigned long long EMPTY64I = 0x000000007FFFFFFFull;
constexpr long long EXT_EMPTY = 0x7FFFFFFFFFFFFFFFll;                  // INT64_MAX (ABI)

template <class T> struct KeyOps;
template <> struct KeyOps<float> {
    using K = unsigned long long;
    static __device__ __forceinline__ void merge(K* p, float v, unsigned i) {
        atomicMin(p, ((K)__float_as_uint(v) << 32) | (K)i);
    }
};
struct alignas(16) K64 { unsigned long long v, i; };
template <> struct KeyOps<double> {
    using K = K64;
    static __device__ __forceinline__ void stage(const K* p, double* thr, unsigned* idx) {
        cp_async8(thr, &p->v);
        cp_async4(idx, &p->i);  // little-endian low word; indices < 2^31
    }
    static __device__ __forceinline__ void merge(K* p, double v, unsigned i) {
        unsigned long long nv = (unsigned long long)__double_as_longlong(v), ni = i;
        ulonglong2 old = __ldcg(reinterpret_cast<const ulonglong2*>(p));
        while (nv < old.x || (nv == old.x && ni < old.y)) {
            unsigned long long ox, oy;
            asm volatile(
                "{\n .reg .b128 c, n, o;\n mov.b128 c, {%2, %3};\n mov.b128 n, {%4, %5};\n"
                " atom.global.cas.b128 o, [%6], c, n;\n mov.b128 {%0, %1}, o;\n}\n"
                : "=l"(ox), "=l"(oy)
                : "l"(old.x), "l"(old.y), "l"(nv), "l"(ni), "l"(p)
                : "memory");
            if (ox == old.x && oy == old.y) break;
            old.x = ox;
            old.y = oy;
        }
    }
};

// Warp OR of a 64-bit mask (two REDUX.OR).
__device__ __forceinline__ unsigned long long or_reduce(unsigned long long v) {
    const unsigned lo = __reduce_or_sync(FULL, (unsigned)v), hi = __reduce_or_sync(FULL, (unsigned)(v >> 32));
    return ((unsigned long long)hi << 32) | lo;
}

// Load the DL dims a lane owns (dims kk*G + g) of one position-major, D-padded row.
template <class T, int DL, int G>
__device__ __forceinline__ void load_dims(const T* __restrict__ rowp, int g, T (&out)[DL]) {
    if constexpr (G == 1 && sizeof(T) == 4 && DL % 4 == 0) {
#pragma unroll
        for (int q = 0; q < DL / 4; ++q) {
            const float4 v = __ldg(reinterpret_cast<const float4*>(rowp) + q);
            out[4 * q] = v.x; out[4 * q + 1] = v.y; out[4 * q + 2] = v.z; out[4 * q + 3] = v.w;
        }
    } else if constexpr (G == 1 && sizeof(T) == 8 && DL % 2 == 0) {
#pragma unroll
        for (int q = 0; q < DL / 2; ++q) {
            const double2 v = __ldg(reinterpret_cast<const double2*>(rowp) + q);
            out[2 * q] = v.x; out[2 * q + 1] = v.y;
        }
    } else {
#pragma unroll
        for (int kk = 0; kk < DL; ++kk) out[kk] = __ldg(rowp + kk * G + g);
    }
}

// ------------------------------------------------------------------ tile order
// Tile t of the launch -> (diagonal block b, row segment q) in the launch's order
// (MainParams::order).  Segment-major: the tiles in flight share their rows and most columns
// (L2 reuse of the staged statistics, faster threshold convergence: C2 FP64 106 -> 91 ms).
// Block-major: the block-cooperative kernels' tiles in flight cover different rows, which
// keeps their lane-local write-through merges off the same keys (segment-major measured
// 1.1-3x slower there: C4 FP64 band 4.3 -> 12.8 s).
__device__ __forceinline__ void decode_tile(const MainParams& p, long long t, int NC, long long& b, long long& q) {
    if (p.order == 1) {
        long long lo = 0, hi = p.nq;
        while (hi - lo > 1) {
            const long long mid = (lo + hi) >> 1;
            if (__ldg(&p.q_prefix[mid]) <= t) lo = mid; else hi = mid;
        }
        q = lo;
        b = __ldg(&p.q_block0[lo]) + (t - __ldg(&p.q_prefix[lo]));
        return;
    }
    t += p.t_begin;
    long long lo = 0, hi = p.nb;
    while (hi - lo > 1) {
        const long long mid = (lo + hi) >> 1;
        if (__ldg(&p.seg_prefix[mid]) <= t) lo = mid; else hi = mid;
    }
    b = lo;
    const long long delta1 = min(p.delta_lo + b * NC + NC - 1, p.delta_hi);
    q = max(max(0ll, -delta1) / p.HT, p.q_lo) + (t - __ldg(&p.seg_prefix[lo]));
}

// ------------------------------------------------------------------ tile geometry
constexpr int pow2ceil(int x) { int p = 1; while (p < x) p <<= 1; return p; }
constexpr int ilog2(int x) { int l = 0; while ((1 << l) < x) ++l; return l; }

template <int G, int W> struct Geo {
    static constexpr int NL = 32 / G;                                   // lane-cells per warp
    // lane-cells per row group: 8 x 4 (rows x lanes) for one cell per lane, else 4 columns
    static constexpr int CA = (W == 1 && NL == 32) ? 8 : (W == 2 && NL == 32) ? MP_CA_W2 : NL >= 16 ? 4 : (NL >= 4 ? 2 : 1);
    static constexpr int RA = NL / CA;                                   // distinct rows per step
    static constexpr int CW = CA * W;                                    // distinct columns per step
    static constexpr int NC = NL * W;                                    // cells (diagonals) per warp
    // ring positions move in batches of SB steps, prefetched one batch ahead: live rows
    // span CW(RA-1) + 2 SB, live columns 2 SB + CW - 1
    static constexpr int SB = G == 1 ? MP_SB_G1 : G == 2 ? MP_SB_G2 : MP_SB_G4;
    static constexpr int RING_R = pow2ceil(CW * (RA - 1) + 2 * SB) < CW ? CW : pow2ceil(CW * (RA - 1) + 2 * SB);
    static constexpr int RPC = RING_R / CW;                              // ring rows per residue class
    static constexpr int RING_C = pow2ceil(2 * SB + CW - 1);
    // plane strides (V4 units): odd for G == 1 so the planes of an entering position hit
    // distinct banks; for G > 1 the G planes read together are shifted by RA (CW) slots.
    static constexpr int PSR = G == 1 ? RING_R + 1 : RING_R + RA;
    static constexpr int PSC = G == 1 ? RING_C + 1 : RING_C + CW;
    static constexpr int LOG_G = ilog2(G), LOG_CA = ilog2(CA), LOG_CW = ilog2(CW), LOG_RPC = ilog2(RPC);
    // ring slot of row r: rows spaced CW apart land in consecutive slots of one class
    static __device__ __forceinline__ int srow(long long r) {
        const int ri = (int)r;
        return ((ri & (CW - 1)) << LOG_RPC) + ((ri >> LOG_CW) & (RPC - 1));
    }
    static __device__ __forceinline__ int scol(long long c) { return (int)c & (RING_C - 1); }
};

template <class T, int DL, int G, int W> struct Smem {
    using V4 = typename PT<T>::V4;
    using Gm = Geo<G, W>;
    static constexpr int D = DL * G;
    static constexpr size_t ring_bytes =
        (((size_t)D * (Gm::PSR + Gm::PSC) * (sizeof(V4) + sizeof(unsigned))) + 15) & ~(size_t)15;
    static constexpr size_t flag_bytes = 0;  // dirty flags live in registers (bit masks)
    static constexpr size_t bytes_per_warp = ring_bytes + flag_bytes + (size_t)W * DL * 32 * sizeof(T);
    // warps per block: up to 4, fewer when a warp's rings are large (blocks <= ~112 KB)
    static constexpr int WPB = bytes_per_warp * 4 <= 112 * 1024 ? 4 : bytes_per_warp * 2 <= 112 * 1024 ? 2 : 1;
};

// plane p holds dimension p's stats in .xyz and, in .w, the threshold of rank
// rank_of_plane(p) -- the rank lane (p % G) holds at register kk = p / G after the sort.
template <int DL, int G> __device__ __forceinline__ int rank_of_plane(int p) { return (p % G) * DL + p / G; }

// ------------------------------------------------------------------ the fused kernel
// minimum resident blocks per SM for the register budget (128 threads per block max)
template <class T, int DL, int G, int W> constexpr int min_blocks() {
    // caps the register budget where ptxas still fits without spills (measured with -Xptxas -v)
    return (sizeof(T) == 4 && G == 1 && DL * W <= 16) ? MP_MINB_F32 : MP_MINB;
}
// COMP: the compensated QT recurrence (reading R4); off for short windows (m < kCompMinM in
// mp_api.cpp), where the plain FP32 recurrence is inside the 1e-4 gate
template <class T, int DL, int G, int W, bool SELF, bool COMP = true>
__global__ void __launch_bounds__(128, (min_blocks<T, DL, G, W>()))
mp_diag(const MainParams p) {
    using V4 = typename PT<T>::V4;
    using Gm = Geo<G, W>;
    using SM = Smem<T, DL, G, W>;
    using KO = KeyOps<T>;
    using K = typename KO::K;
    constexpr int CA = Gm::CA, RA = Gm::RA, CW = Gm::CW, D = DL * G;
    constexpr int PSR = Gm::PSR, PSC = Gm::PSC;
    constexpr int SB = Gm::SB;
    constexpr int FOLD = SB > MP_FOLD ? SB : MP_FOLD;  // steps between folds of QL into QT

    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned char* wbase = smem_raw + (size_t)warp * SM::bytes_per_warp;
    V4* rowv = reinterpret_cast<V4*>(wbase);
    V4* colv = rowv + (size_t)D * PSR;
    // ring keys: the warp's current (value, index) best of each staged (position, rank), the
    // index word's bit 31 marking it dirty; the .w words are filter hints only
    // ring indices: the index of the warp's own best (value in the slot's .w) of a staged
    // (position, rank), DIRTY when it improved on the staged global key; EMPTY_IDX until then.
    // Only locally found indices live here -- the global key's index is never staged, so a key
    // updated by another warp between its value and index reads cannot pair a value with a
    // foreign index (a tie with the staged value is taken locally and settled by the merge).
    unsigned* rowi = reinterpret_cast<unsigned*>(colv + (size_t)D * PSC);
    unsigned* coli = rowi + (size_t)D * PSR;
    // dirty ring slots: warp-uniform bit masks in registers (slot -> bit), set after each
    // slow path by a warp OR-reduction, cleared on eviction -- no shared-memory flags to poll
    static_assert(Gm::RING_R <= 64 && Gm::RING_C <= 64, "dirty masks hold one bit per ring slot");
    using DMask = unsigned long long;
    DMask dmask_r = 0, dmask_c = 0;
    T* ssc = reinterpret_cast<T*>(wbase + SM::ring_bytes + SM::flag_bytes);

    const V4* __restrict__ st_q = reinterpret_cast<const V4*>(p.st_q);
    const V4* __restrict__ st_r = reinterpret_cast<const V4*>(p.st_r);
    const T* __restrict__ tw_q = reinterpret_cast<const T*>(p.tw_q);
    const T* __restrict__ tw_r = reinterpret_cast<const T*>(p.tw_r);
    const T* __restrict__ mu_q = reinterpret_cast<const T*>(p.mu_q);
    const T* __restrict__ mu_r = reinterpret_cast<const T*>(p.mu_r);
    K* keys = reinterpret_cast<K*>(p.keys);

    const long long n = p.n;
    const int d = p.d, m = p.m, H = p.H, HT = p.HT;
    const T two_m = (T)(2 * m);
    const T INF = PT<T>::inf(), NINF = PT<T>::ninf();

    const int lc = lane >> Gm::LOG_G, g = lane & (G - 1);
    const int a = lc >> Gm::LOG_CA, c = lc & (CA - 1);
    // lanes of the same row group (same a, g) vary c; same column group (c, g) vary a
    unsigned gmask_row = 0, gmask_col = 0;
#pragma unroll
    for (int cc = 0; cc < CA; ++cc) gmask_row |= 1u << (((a * CA + cc) << Gm::LOG_G) + g);
#pragma unroll
    for (int aa = 0; aa < RA; ++aa) gmask_col |= 1u << (((aa * CA + c) << Gm::LOG_G) + g);

    // --- ring staging.  Positions move through the rings in batches of SB steps:
    // stage() starts the async copies (cp.async / LDGSTS) of a range of entering positions'
    // stats (.xyz), thresholds (.w = the value half of the merge key) and best indices one
    // batch ahead; evict() merges positions whose ring copy improved (dirty) into global
    // memory.  The (position, plane) pairs of a range are spread over the 32 lanes.
    const int n32 = (int)n;
    auto stage = [&](bool is_row, int base, int p_lo, int p_hi) {
        const int cnt = p_hi - p_lo;
        if (cnt <= 0) return;
        V4* buf = is_row ? rowv : colv;
        unsigned* ib = is_row ? rowi : coli;
        const int ps = is_row ? PSR : PSC;
        const V4* __restrict__ st = is_row ? st_q : st_r;
        const bool want_thr = is_row || SELF;
        if (d == D && base + p_lo >= 0 && base + p_hi <= n32 && want_thr) {
            // common case: all positions in range, no padded dims -- branch-free copies
            for (int e = lane; e < cnt * D; e += 32) {
                const int pi = e / D, pl = e - pi * D;
                const int pos = base + p_lo + pi;
                const int sl = is_row ? Gm::srow(pos) : Gm::scol(pos);
                V4* dst = &buf[pl * ps + sl];
                const V4* src = st + (size_t)pos * d + pl;
                if constexpr (sizeof(T) == 4) {
                    cp_async8(dst, src);
                    cp_async4(&dst->z, &src->z);
                } else {
                    cp_async16(dst, src);
                    cp_async8(&dst->z, &src->z);
                }
                cp_async4(&dst->w, reinterpret_cast<const char*>(keys + (size_t)pos * d + rank_of_plane<DL, G>(pl)) + 4);
                ib[pl * ps + sl] = EMPTY_IDX;
            }
            return;
        }
        for (int e = lane; e < cnt * D; e += 32) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            if (pos < 0 || pos >= n32) continue;
            const int sl = is_row ? Gm::srow(pos) : Gm::scol(pos);
            V4* dst = &buf[pl * ps + sl];
            const V4* src = st + (size_t)pos * d + pl;
            if (pl < d) {
                if constexpr (sizeof(T) == 4) {
                    cp_async8(dst, src);                      // df, dg
                    cp_async4(&dst->z, &src->z);              // a
                } else {
                    cp_async16(dst, src);
                    cp_async8(&dst->z, &src->z);
                }
            } else {  // padded dimension: a = pad_a with QT = -1 gives D ~ 1e18 (sorts last)
                dst->x = 0; dst->y = 0; dst->z = PT<T>::pad_a();
            }
            const int rk = rank_of_plane<DL, G>(pl);
            if (rk < d && want_thr) {
                cp_async4(&dst->w, reinterpret_cast<const char*>(keys + (size_t)pos * d + rk) + 4);
                ib[pl * ps + sl] = EMPTY_IDX;
            } else {
                dst->w = NINF;  // never hit
                ib[pl * ps + sl] = EMPTY_IDX;
            }
        }
    };
    auto evict = [&](bool is_row, int base, int p_lo, int p_hi) {
        if (!is_row && !SELF) return;
        const int cnt = p_hi - p_lo;
        if (cnt <= 0) return;
        const V4* buf = is_row ? rowv : colv;
        const unsigned* ib = is_row ? rowi : coli;
        const int ps = is_row ? PSR : PSC;
        // early out (warp-uniform, registers only): most evictions find nothing dirty
        DMask& dm = is_row ? dmask_r : dmask_c;
        if (dm == 0) return;
        DMask leaving = 0;
        for (int pi = 0; pi < cnt; ++pi) {
            const int pos = base + p_lo + pi;
            leaving |= 1ull << (is_row ? Gm::srow(pos) : Gm::scol(pos));
        }
        const DMask dirty = dm & leaving;
        if (dirty == 0) return;
        dm &= ~leaving;
        for (int e = lane; e < cnt * D; e += 32) {
            const int pi = e / D, pl = e - pi * D;
            const int pos = base + p_lo + pi;
            if (pos < 0 || pos >= n32) continue;
            const int sl = is_row ? Gm::srow(pos) : Gm::scol(pos);
            if (((dirty >> sl) & 1ull) == 0) continue;
            const int rk = rank_of_plane<DL, G>(pl);
            if (rk >= d) continue;
            const unsigned kv = ib[pl * ps + sl];
            if (kv & DIRTY)   // the slot's .w is the value of the warp's best (set with the index)
                atomicMin(keys + (size_t)pos * d + rk, ((K)__float_as_uint(buf[pl * ps + sl].w) << 32) | (kv & ~DIRTY));
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

        // the lane's W cells: diagonals and valid row ranges inside the tile
        long long delta[W], lo[W], hi[W];
#pragma unroll
        for (int u = 0; u < W; ++u) {
            delta[u] = delta0 + (long long)a * CW + c * W + u;
            lo[u] = max(r0, max(0ll, -delta[u]));
            hi[u] = min(r1, n - max(delta[u], 0ll));
            if (delta[u] > p.delta_hi) hi[u] = lo[u];
        }
        int dlt[W], lo32[W], hi32[W];  // positions and diagonals fit in 32 bits (n < 2^31)
#pragma unroll
        for (int u = 0; u < W; ++u) { dlt[u] = (int)delta[u]; lo32[u] = (int)lo[u]; hi32[u] = (int)hi[u]; }

        // seeds: direct centred dot products (reading G8), compensated
        // (Kahan) accumulation, at each cell's first row and then every H rows (reseed(),
        // called at warp-uniform steps; the tile is HT >= H rows tall).  Operands are
        // position-major and padded to D dims, so a lane (G == 1) loads its DL dims as vectors.
        // QT = QT[u][kk] + QL[u][kk] (compensated, reading R4): increments accumulate into the
        // small word QL, which is folded into QT by an exact Fast2Sum every FOLD steps
        T QT[W][DL], QL[W][DL];
        auto seed_cell = [&](int u, long long row) {
            // dims in chunks of SC: the m-long dot-product loop then keeps few operand
            // registers live, so seeding never sets the kernel's register peak
            constexpr int SC = (DL % MP_SEED_CHUNK == 0) ? MP_SEED_CHUNK : DL;
            const long long i0 = row, j0 = row + delta[u];
            const T* xq_p = tw_q + i0 * D;
            const T* xr_p = tw_r + j0 * D;
#pragma unroll
            for (int c0 = 0; c0 < DL; c0 += SC) {
                T mq[SC], mr[SC], cmp[SC], acc[SC];
                load_dims<T, SC, G>(mu_q + i0 * D + c0 * G, g, mq);
                load_dims<T, SC, G>(mu_r + j0 * D + c0 * G, g, mr);
#pragma unroll
                for (int kk = 0; kk < SC; ++kk) { acc[kk] = (T)0; cmp[kk] = (T)0; }
#pragma unroll 2
                for (int tt = 0; tt < m; ++tt) {
                    T xq[SC], xr[SC];
                    load_dims<T, SC, G>(xq_p + (long long)tt * D + c0 * G, g, xq);
                    load_dims<T, SC, G>(xr_p + (long long)tt * D + c0 * G, g, xr);
#pragma unroll
                    for (int kk = 0; kk < SC; ++kk) {
                        const T y = (xq[kk] - mq[kk]) * (xr[kk] - mr[kk]) - cmp[kk];
                        const T t2 = acc[kk] + y;
                        cmp[kk] = (t2 - acc[kk]) - y;
                        acc[kk] = t2;
                    }
                }
#pragma unroll
                for (int kk = 0; kk < SC; ++kk) {  // the Kahan sum is acc - cmp: keep both words
                    const bool pad = ((c0 + kk) * G + g) >= d;  // padded dims: zero data
                    QT[u][c0 + kk] = pad ? (T)-1 : (COMP ? acc[kk] : acc[kk] - cmp[kk]);
                    QL[u][c0 + kk] = pad ? (T)0 : (COMP ? -cmp[kk] : (T)0);
                }
            }
        };
#pragma unroll
        for (int u = 0; u < W; ++u) {
            if (lo[u] < hi[u]) {
                seed_cell(u, lo[u]);
            } else {
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) { QT[u][kk] = (kk * G + g) >= d ? (T)-1 : (T)0; QL[u][kk] = (T)0; }
            }
        }
        int seeded_step = -1;  // step whose row was re-seeded at its batch start
        dmask_r = 0;
        dmask_c = 0;

        const int nrows = (int)(r1 - r0);
        const int s_end = nrows + CW * (RA - 1);
        const int R0 = (int)r0, C0 = (int)(r0 + delta0);  // row / column of step 0, cell 0
        // batch pipeline bookkeeping (positions relative to R0 / C0)
        int row_in = min(SB, nrows), col_in = min(SB, s_end) + CW - 1, row_out = 0, col_out = 0;
        stage(true, R0, 0, row_in);
        stage(false, C0, 0, col_in);
        cp_async_commit();
        cp_async_wait_all();
        __syncwarp();

        // W == 2: column data of cell u = 0 is carried from cell u = 1 of the previous step
        constexpr int CD = W == 2 ? DL : 1;
        V4 carA[CD], carB[CD];
        if constexpr (W == 2) {
            const int sc0 = Gm::scol(C0 + c * W);
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) carA[kk] = colv[kk * PSC + sc0];
        }

        // one step: cells (row, row + delta[u]) of this lane
        auto step = [&](int s, V4 (&Cold)[CD], V4 (&Cnew)[CD]) {
            const int row = R0 + s - CW * a;
            const int sr = Gm::srow(row);
            bool active[W], upd[W];
            int col[W];
#pragma unroll
            for (int u = 0; u < W; ++u) {
                col[u] = row + dlt[u];
                active[u] = row >= lo32[u] && row < hi32[u];
                upd[u] = row > lo32[u] && row < hi32[u];
            }
            if (s == seeded_step) {  // QT of this row was just seeded
#pragma unroll
                for (int u = 0; u < W; ++u) upd[u] = false;
            }
            const int scn = Gm::scol(col[W - 1]);

            // thresholds stay in registers for small per-lane dim counts; wide lanes
            // re-read them from the ring after the sort (register budget)
            constexpr bool KEEP = (DL * W <= MP_KEEP_DL);
            T S[W][DL], tr[KEEP ? DL : 1], tc0[KEEP ? DL : 1];
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) {
                const int pl = kk * G + g;
                const V4 R = rowv[pl * PSR + sr];
                const V4 C = colv[pl * PSC + scn];
                if constexpr (W == 2) {
                    const V4 C0v = Cold[kk];
                    const T pr0 = R.z * C0v.z;
                    if constexpr (COMP) {
                        if (upd[0]) QL[0][kk] = fma(R.x, C0v.y, fma(C0v.x, R.y, QL[0][kk]));   // Eq. (1)
                        S[0][kk] = PT<T>::sqrt_abs(fma(-QL[0][kk], pr0, fma(-QT[0][kk], pr0, two_m)));
                    } else {
                        if (upd[0]) QT[0][kk] = fma(R.x, C0v.y, fma(C0v.x, R.y, QT[0][kk]));   // Eq. (1)
                        S[0][kk] = PT<T>::sqrt_abs(fma(-QT[0][kk], pr0, two_m));
                    }
                    if constexpr (KEEP) tc0[kk] = C0v.w;
                    Cnew[kk] = C;
                }
                const T pr = R.z * C.z;
                if constexpr (COMP) {
                    if (upd[W - 1]) QL[W - 1][kk] = fma(R.x, C.y, fma(C.x, R.y, QL[W - 1][kk]));  // Eq. (1)
                    S[W - 1][kk] = PT<T>::sqrt_abs(fma(-QL[W - 1][kk], pr, fma(-QT[W - 1][kk], pr, two_m)));  // Eq. (1)
                } else {
                    if (upd[W - 1]) QT[W - 1][kk] = fma(R.x, C.y, fma(C.x, R.y, QT[W - 1][kk]));  // Eq. (1)
                    S[W - 1][kk] = PT<T>::sqrt_abs(fma(-QT[W - 1][kk], pr, two_m));                // Eq. (1)
                }
                if constexpr (KEEP) {
                    tr[kk] = R.w;
                    if constexpr (W == 1) tc0[kk] = C.w;
                }
            }
#pragma unroll
            for (int u = 0; u < W; ++u) {
                if constexpr (G == 1 && MP_FUSE_LAST && DL >= 8 && last_layer_adjacent<DL>()) {
                    sort_scan_fused<T, DL>(S[u]);                                     // Eq. (2) sort + scan
                } else {
                sort_net<T, DL>(S[u]);                                               // Eq. (2) sort
                if (G > 1) lane_merge<T, DL, G>(S[u], g);
                // Eq. (2) inclusive scan, two independent half chains joined at the end
                // (shorter dependency chain; summation order differs only by rounding)
                if constexpr (DL >= 8) {
#pragma unroll
                    for (int kk = 1; kk < DL / 2; ++kk) S[u][kk] += S[u][kk - 1];
#pragma unroll
                    for (int kk = DL / 2 + 1; kk < DL; ++kk) S[u][kk] += S[u][kk - 1];
#pragma unroll
                    for (int kk = DL / 2; kk < DL; ++kk) S[u][kk] += S[u][DL / 2 - 1];
                } else {
#pragma unroll
                    for (int kk = 1; kk < DL; ++kk) S[u][kk] += S[u][kk - 1];
                }
                }
                if (G > 1) {
                    T tot = S[u][DL - 1];
#pragma unroll
                    for (int dd = 1; dd < G; dd <<= 1) {
                        T y = __shfl_up_sync(FULL, tot, dd, G);
                        if (g >= dd) tot += y;
                    }
                    T excl = __shfl_up_sync(FULL, tot, 1, G);
                    if (g == 0) excl = (T)0;
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) S[u][kk] += excl;
                }
            }
            bool hit = false;
#pragma unroll
            for (int u = 0; u < W; ++u) {
                bool h[4] = {false, false, false, false};  // independent predicate chains (ILP)
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    if constexpr (KEEP) {
                        h[kk & 3] |= S[u][kk] <= tr[kk];
                        if (SELF) {
                            if constexpr (W == 2) h[kk & 3] |= S[u][kk] <= (u == 0 ? tc0[kk] : Cnew[kk].w);
                            else h[kk & 3] |= S[u][kk] <= tc0[kk];
                        }
                    } else {
                        const int pl = kk * G + g;
                        h[kk & 3] |= S[u][kk] <= rowv[pl * PSR + sr].w;
                        if (SELF) h[kk & 3] |= S[u][kk] <= colv[pl * PSC + Gm::scol(col[u])].w;
                    }
                }
                hit |= ((h[0] | h[1]) | (h[2] | h[3])) && active[u];
            }
            if (__any_sync(FULL, hit)) {
                // Eq. (3) with the lowest-index tie rule: group min by shuffles, one leader
                // per row / column group compares (value, index) with the ring's best.
                DMask mark_r = 0, mark_c = 0;  // ring slots this lane's leader updates dirtied
                auto rank_update = [&](const int kk, const T (&v)[W]) {
                    const int pl = kk * G + g;
                    // skip ranks (and sides) no lane can improve: most slow steps touch 1-2 ranks
                    T vmin_l = v[0];
#pragma unroll
                    for (int u = 1; u < W; ++u) vmin_l = PT<T>::vmin(vmin_l, v[u]);
                    const bool need_r = __any_sync(FULL, vmin_l <= rowv[pl * PSR + sr].w);
                    bool need_c = false;
                    if (SELF) {
#pragma unroll
                        for (int u = 0; u < W; ++u) need_c |= v[u] <= colv[pl * PSC + Gm::scol(col[u])].w;
                        need_c = __any_sync(FULL, need_c);
                    }
                    if (!need_r && !need_c) return;
                    __syncwarp();   // every lane read the ring bests before a leader updates them
                    // row group: W cells per lane x CA lanes
                    T vr = v[0];
#pragma unroll
                    for (int u = 1; u < W; ++u) vr = PT<T>::vmin(vr, v[u]);
#pragma unroll
                    for (int bit = 0; bit < Gm::LOG_CA; ++bit)
                        vr = PT<T>::vmin(vr, __shfl_xor_sync(FULL, vr, 1 << (bit + Gm::LOG_G)));
                    bool mine = false;
#pragma unroll
                    for (int u = 0; u < W; ++u) mine |= v[u] == vr;
                    const unsigned eqr = __ballot_sync(FULL, mine) & gmask_row;
                    if (need_r && vr < INF && lane == __ffs(eqr) - 1) {
                        int j = col[W - 1];
#pragma unroll
                        for (int u = W - 1; u >= 0; --u)
                            if (v[u] == vr) j = col[u];                 // lowest column first
                        const int ix = pl * PSR + sr;
                        const T cur = rowv[ix].w;
                        const unsigned ci = rowi[ix] & ~DIRTY;
                        if (vr < cur || (vr == cur && (unsigned)j < ci)) {
                            rowv[ix].w = vr;
                            rowi[ix] = (unsigned)j | DIRTY;
                            mark_r |= 1ull << sr;
                        }
                    }
                    if (SELF && need_c) {
#pragma unroll
                        for (int u = 0; u < W; ++u) {
                            T vc = v[u];
#pragma unroll
                            for (int bit = 0; bit < 5 - Gm::LOG_G - Gm::LOG_CA; ++bit)
                                vc = PT<T>::vmin(vc, __shfl_xor_sync(FULL, vc, 1 << (bit + Gm::LOG_G + Gm::LOG_CA)));
                            const unsigned eqc = __ballot_sync(FULL, v[u] == vc) & gmask_col;
                            // lowest row index = highest a = highest lane
                            if (vc < INF && eqc != 0 && lane == 31 - __clz(eqc)) {
                                const int scu = Gm::scol(col[u]);
                                const int ix = pl * PSC + scu;
                                const T cur = colv[ix].w;
                                const unsigned ci = coli[ix] & ~DIRTY;
                                if (vc < cur || (vc == cur && (unsigned)row < ci)) {
                                    colv[ix].w = vc;
                                    coli[ix] = (unsigned)row | DIRTY;
                                    mark_c |= 1ull << scu;
                                }
                            }
                        }
                    }
                    __syncwarp();   // the leaders' ring updates are visible to the next rank's reads
                };
                if constexpr (MP_SLOW_UNROLL) {
                    // ranks some lane can improve, from registers (S stays live; the ring's
                    // current bests are re-read); then a fully unrolled pass over the ranks
                    // with a warp-uniform skip: no shared-memory round trip of S
                    unsigned rk_bits = 0;
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) {
                        const int pl = kk * G + g;
                        const T tr_k = rowv[pl * PSR + sr].w;
                        bool hk = false;
#pragma unroll
                        for (int u = 0; u < W; ++u) {
                            hk |= active[u] && S[u][kk] <= tr_k;
                            if (SELF) hk |= active[u] && S[u][kk] <= colv[pl * PSC + Gm::scol(col[u])].w;
                        }
                        rk_bits |= (unsigned)hk << kk;
                    }
                    rk_bits = __reduce_or_sync(FULL, rk_bits);
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) {
                        if (!((rk_bits >> kk) & 1u)) continue;
                        T v[W];
#pragma unroll
                        for (int u = 0; u < W; ++u) v[u] = active[u] ? S[u][kk] : INF;
                        rank_update(kk, v);
                    }
                } else {
#pragma unroll
                for (int u = 0; u < W; ++u)
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) ssc[(u * DL + kk) * 32 + lane] = active[u] ? S[u][kk] : INF;
                __syncwarp();
                // ranks some lane can improve (compared with the current ring bests, from
                // shared memory so no register stays live across the slow path): one warp OR,
                // then the loop visits only those ranks -- a slow step touches 1-2 of DL ranks
                unsigned rk_bits = 0;
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) {
                    const int pl = kk * G + g;
                    const T tr_k = rowv[pl * PSR + sr].w;
                    bool hk = false;
#pragma unroll
                    for (int u = 0; u < W; ++u) {
                        const T v = ssc[(u * DL + kk) * 32 + lane];
                        hk |= v <= tr_k;
                        if (SELF) hk |= v <= colv[pl * PSC + Gm::scol(col[u])].w;
                    }
                    rk_bits |= (unsigned)hk << kk;
                }
                rk_bits = __reduce_or_sync(FULL, rk_bits);
#pragma unroll 1
                for (; rk_bits != 0; rk_bits &= rk_bits - 1) {
                    const int kk = __ffs(rk_bits) - 1;
                    T v[W];
#pragma unroll
                    for (int u = 0; u < W; ++u) v[u] = ssc[(u * DL + kk) * 32 + lane];
                    rank_update(kk, v);
                }
                }
                dmask_r |= or_reduce(mark_r);
                dmask_c |= or_reduce(mark_c);
                __syncwarp();
            }
        };

        int to_seed = H;  // steps until the next re-seed (H is a multiple of SB)
        for (int s0 = 0; s0 < s_end; s0 += SB) {
            if (COMP && (s0 & (FOLD - 1)) == 0) {  // fold the increments into QT (exact Fast2Sum)
#pragma unroll
                for (int u = 0; u < W; ++u)
#pragma unroll
                    for (int kk = 0; kk < DL; ++kk) {
                        const T t = QT[u][kk] + QL[u][kk];
                        QL[u][kk] = QL[u][kk] - (t - QT[u][kk]);
                        QT[u][kk] = t;
                    }
            }
            // seeds: each cell's first row at s0 = 0, then the current row every H steps
            // (H is a multiple of SB, so re-seeds fall on batch starts: one call site)
            if (s0 > 0 && (to_seed -= SB) == 0) {
                to_seed = H;
                const long long row = R0 + s0 - (long long)CW * a;
#pragma unroll 1
                for (int u = 0; u < W; ++u)
                    if (row > lo[u] && row < hi[u]) seed_cell(u, row);
                seeded_step = s0;
            }
            // evict positions no step from s0 on reads; prefetch the next batch's entries
            const int rx = min(max(s0 - CW * (RA - 1), 0), nrows);
            evict(true, R0, row_out, rx);
            row_out = rx;
            evict(false, C0, col_out, s0);
            col_out = s0;
            __syncwarp();   // every eviction read its ring slot before a prefetch can overwrite it
            const int nxt = min(s0 + 2 * SB, s_end);
            const int r_need = min(nxt, nrows), c_need = nxt + CW - 1;
            stage(true, R0, row_in, r_need);
            stage(false, C0, col_in, c_need);
            row_in = max(row_in, r_need);
            col_in = max(col_in, c_need);
            cp_async_commit();
            if constexpr (W == 2) {  // ping-pong the carried column registers (no moves)
#pragma unroll 1
                for (int k2 = 0; k2 < SB; k2 += 2) {
                    if (s0 + k2 < s_end) step(s0 + k2, carA, carB);
                    if (s0 + k2 + 1 < s_end) step(s0 + k2 + 1, carB, carA);
                }
            } else {  // one copy of the step body (instruction-cache footprint)
                const int s1 = min(s0 + SB, s_end);
                MP_UNROLL(MP_W1_UNROLL)
                for (int ss = s0; ss < s1; ++ss) step(ss, carA, carB);
            }
            cp_async_wait_all();   // this lane's prefetch for the next batch has landed
            __syncwarp();          // ... and everyone's; all reads of this batch are done
        }
        // epilogue: evict what is still in the rings
        evict(true, R0, row_out, nrows);
        evict(false, C0, col_out, col_in);
        __syncwarp();
    }
}

template <class T, int DL, int G, int W, bool SELF, bool COMP = true> struct Inst {
    static size_t smem();
    static cudaError_t launch(const MainParams& p, int grid, cudaStream_t s);
    static int blocks_per_sm();
    static int warps_per_block() { return Smem<T, DL, G, W>::WPB; }
};

#ifdef MP_DIAG_IMPL
template <class T, int DL, int G, int W, bool SELF, bool COMP> size_t Inst<T, DL, G, W, SELF, COMP>::smem() {
    return Smem<T, DL, G, W>::bytes_per_warp * Smem<T, DL, G, W>::WPB;
}
template <class T, int DL, int G, int W, bool SELF, bool COMP>
cudaError_t Inst<T, DL, G, W, SELF, COMP>::launch(const MainParams& p, int grid, cudaStream_t s) {
    const size_t sm = smem();
    cudaError_t e = cudaFuncSetAttribute(mp_diag<T, DL, G, W, SELF, COMP>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    mp_diag<T, DL, G, W, SELF, COMP><<<grid, Smem<T, DL, G, W>::WPB * 32, sm, s>>>(p);
    return cudaGetLastError();
}
template <class T, int DL, int G, int W, bool SELF, bool COMP> int Inst<T, DL, G, W, SELF, COMP>::blocks_per_sm() {
    const size_t sm = smem();
    cudaFuncSetAttribute(mp_diag<T, DL, G, W, SELF, COMP>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    int nb = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, mp_diag<T, DL, G, W, SELF, COMP>, Smem<T, DL, G, W>::WPB * 32, sm);
    return nb;
}
#endif

}  // namespace mpk

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
//   cell when d > 32 (each holds DL dims); the NC cells of a warp step are arranged as
//   RA rows x CA columns (row = r0 + s - CA*a, col = row + delta) so a step touches
//   RA distinct rows and CA distinct columns.  Row/column statistics and the running
//   profile thresholds are staged in per-warp shared-memory rings (rows enter once per
//   step, leave after RA*CA steps), so the inner loop reads 2 LDS per cell-dim.  The
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

namespace mpk {

constexpr unsigned FULL = 0xffffffffu;
constexpr int WARPS_PER_BLOCK = 4;
constexpr unsigned DIRTY = 0x80000000u;

// ------------------------------------------------------------------ precision traits
template <class T> struct PT;
template <> struct PT<float> {
    using V4 = float4;
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

// Batcher odd-even merge sort network on N registers (any N; fully unrolled at compile
// time).  Ascending (Eq. 2 "sort", reading G12).
template <class T, int N> __device__ __forceinline__ void sort_net(T (&v)[N]) {
#pragma unroll
    for (int p = 1; p < N; p <<= 1) {
#pragma unroll
        for (int k = p; k >= 1; k >>= 1) {
#pragma unroll
            for (int j = k % p; j + k < N; j += 2 * k) {
#pragma unroll
                for (int i = 0; i < k; ++i) {
                    if (i + j + k < N && (i + j) / (2 * p) == (i + j + k) / (2 * p)) cswap(v[i + j], v[i + j + k]);
                }
            }
        }
    }
}

// Bitonic merge of the sorted DL-blocks held by G consecutive lanes (lane-blocked order:
// lane g ends up with ranks [g*DL, (g+1)*DL)).  The paper's group-cooperative bitonic
// sort expressed with warp shuffles instead of shared memory.
template <class T, int DL, int G> __device__ __forceinline__ void lane_merge(T (&v)[DL], int g) {
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
        for (int dist = DL / 2; dist >= 1; dist >>= 1) {
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
constexpr unsigned long long EMPTY32 = 0x7F800000FFFFFFFFull;          // (+inf, 2^32-1)
constexpr unsigned long long EMPTY64V = 0x7FF0000000000000ull;         // +inf
constexpr unsigned long long EMPTY64I = 0x7FFFFFFFFFFFFFFFull;

template <class T> struct KeyOps;
template <> struct KeyOps<float> {
    using K = unsigned long long;
    static __device__ __forceinline__ void load(const K* p, float& v, unsigned& i) {
        K k = __ldcg(p);
        v = __uint_as_float((unsigned)(k >> 32));
        i = (unsigned)k;
    }
    static __device__ __forceinline__ void merge(K* p, float v, unsigned i) {
        atomicMin(p, ((K)__float_as_uint(v) << 32) | (K)i);
    }
};
struct alignas(16) K64 { unsigned long long v, i; };
template <> struct KeyOps<double> {
    using K = K64;
    static __device__ __forceinline__ void load(const K* p, double& v, unsigned& i) {
        ulonglong2 k = __ldcg(reinterpret_cast<const ulonglong2*>(p));
        v = __longlong_as_double((long long)k.x);
        i = (k.y > 0xffffffffull) ? 0xffffffffu : (unsigned)k.y;
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

// ------------------------------------------------------------------ tile geometry
template <int G> struct Geo {
    static constexpr int NC = 32 / G;                                   // cells per warp step
    static constexpr int CA = NC >= 16 ? 4 : (NC >= 4 ? 2 : 1);         // distinct columns per step
    static constexpr int RA = NC / CA;                                   // distinct rows per step
    static constexpr int LIVE_R = CA * (RA - 1) + 2;
    static constexpr int RING_R0 = LIVE_R <= 2 ? 2 : LIVE_R <= 4 ? 4 : LIVE_R <= 8 ? 8 : LIVE_R <= 16 ? 16 : 32;
    static constexpr int RING_R = RING_R0 < 8 ? 8 : RING_R0;
    static constexpr int RPC = RING_R / CA;                              // ring rows per residue class
    static constexpr int RING_C = (2 * CA) < 8 ? 8 : 2 * CA;
    static constexpr int PSR = RING_R + RA;                              // plane stride (elements), padded
    static constexpr int PSC = RING_C + CA;
    static constexpr int LOG_G = G == 1 ? 0 : G == 2 ? 1 : G == 4 ? 2 : G == 8 ? 3 : G == 16 ? 4 : 5;
    static constexpr int LOG_CA = CA == 1 ? 0 : CA == 2 ? 1 : 2;
    // ring slot of row r: rows spaced CA apart land in consecutive slots of one class
    static __device__ __forceinline__ int srow(long long r) {
        int ri = (int)r;
        return (ri & (CA - 1)) * RPC + ((ri >> LOG_CA) & (RPC - 1));
    }
    static __device__ __forceinline__ int scol(long long c) { return (int)c & (RING_C - 1); }
};

template <class T, int DL, int G> struct Smem {
    using V4 = typename PT<T>::V4;
    using Gm = Geo<G>;
    static constexpr int D = DL * G;
    static constexpr size_t ring_bytes =
        (((size_t)D * (Gm::PSR + Gm::PSC) * (sizeof(V4) + sizeof(unsigned))) + 15) & ~(size_t)15;
    static constexpr size_t bytes_per_warp = ring_bytes + (size_t)DL * 32 * sizeof(T);  // + slow-path scratch
};

// plane p holds dimension p's stats in .xyz and, in .w, the threshold of rank
// rank_of_plane(p) -- the rank lane (p % G) holds at register kk = p / G after the sort.
template <int DL, int G> __device__ __forceinline__ int rank_of_plane(int p) { return (p % G) * DL + p / G; }

// ------------------------------------------------------------------ the fused kernel
template <class T, int DL, int G, bool SELF>
__global__ void __launch_bounds__(WARPS_PER_BLOCK * 32)
mp_diag(const MainParams p) {
    using V4 = typename PT<T>::V4;
    using Gm = Geo<G>;
    using KO = KeyOps<T>;
    using K = typename KO::K;
    constexpr int NC = Gm::NC, CA = Gm::CA, RA = Gm::RA, D = DL * G;
    constexpr int PSR = Gm::PSR, PSC = Gm::PSC;

    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    unsigned char* wbase = smem_raw + (size_t)warp * Smem<T, DL, G>::bytes_per_warp;
    V4* rowv = reinterpret_cast<V4*>(wbase);
    V4* colv = rowv + (size_t)D * PSR;
    unsigned* rowi = reinterpret_cast<unsigned*>(colv + (size_t)D * PSC);
    unsigned* coli = rowi + (size_t)D * PSR;
    T* ssc = reinterpret_cast<T*>(wbase + Smem<T, DL, G>::ring_bytes);

    const V4* __restrict__ st_q = reinterpret_cast<const V4*>(p.st_q);
    const V4* __restrict__ st_r = reinterpret_cast<const V4*>(p.st_r);
    const T* __restrict__ tw_q = reinterpret_cast<const T*>(p.tw_q);
    const T* __restrict__ tw_r = reinterpret_cast<const T*>(p.tw_r);
    const T* __restrict__ mu_q = reinterpret_cast<const T*>(p.mu_q);
    const T* __restrict__ mu_r = reinterpret_cast<const T*>(p.mu_r);
    K* keys = reinterpret_cast<K*>(p.keys);

    const long long n = p.n;
    const int d = p.d, m = p.m, H = p.H;
    const long long L = n + m - 1;
    const T two_m = (T)(2 * m);
    const T INF = PT<T>::inf(), NINF = PT<T>::ninf();

    const int cell = lane >> Gm::LOG_G, g = lane & (G - 1);
    const int a = cell >> Gm::LOG_CA, c = cell & (CA - 1);
    // lanes of the same row group (same a, g): vary c; same column group (c, g): vary a
    const unsigned gmask_row = [&] {
        unsigned mk = 0;
        for (int cc = 0; cc < CA; ++cc) mk |= 1u << (((a * CA + cc) << Gm::LOG_G) + g);
        return mk;
    }();
    const unsigned gmask_col = [&] {
        unsigned mk = 0;
        for (int aa = 0; aa < RA; ++aa) mk |= 1u << (((aa * CA + c) << Gm::LOG_G) + g);
        return mk;
    }();

    // --- ring staging helpers (each lane handles planes lane, lane+32, ...)
    auto enter = [&](bool is_row, long long pos, const V4* __restrict__ st) {
        if (pos < 0 || pos >= n) return;
        V4* buf = is_row ? rowv : colv;
        unsigned* ib = is_row ? rowi : coli;
        const int ps = is_row ? PSR : PSC;
        const int sl = is_row ? Gm::srow(pos) : Gm::scol(pos);
        for (int pl = lane; pl < D; pl += 32) {
            V4 v;
            if (pl < d) {
                v = st[pos * d + pl];
            } else {  // padded dimension: a = +inf with QT = -1 gives D = +inf (sorts last)
                v.x = 0; v.y = 0; v.z = INF;
            }
            const int rk = rank_of_plane<DL, G>(pl);
            unsigned ix = 0;
            T thr = NINF;  // never hit
            if (rk < d && (is_row || SELF)) KO::load(keys + pos * d + rk, thr, ix);
            v.w = thr;
            buf[pl * ps + sl] = v;
            ib[pl * ps + sl] = ix & ~DIRTY;
        }
    };
    auto leave = [&](bool is_row, long long pos) {
        if (pos < 0 || pos >= n) return;
        if (!is_row && !SELF) return;
        const V4* buf = is_row ? rowv : colv;
        const unsigned* ib = is_row ? rowi : coli;
        const int ps = is_row ? PSR : PSC;
        const int sl = is_row ? Gm::srow(pos) : Gm::scol(pos);
        for (int pl = lane; pl < D; pl += 32) {
            const int rk = rank_of_plane<DL, G>(pl);
            if (rk >= d) continue;
            const unsigned ix = ib[pl * ps + sl];
            if (ix & DIRTY) KO::merge(keys + pos * d + rk, buf[pl * ps + sl].w, ix & ~DIRTY);
        }
    };

    for (;;) {
        long long t = 0;
        if (lane == 0) t = (long long)atomicAdd(p.counter, 1ull);
        t = __shfl_sync(FULL, t, 0);
        if (t >= p.t_count) break;
        t += p.t_begin;
        // block b: seg_prefix[b] <= t < seg_prefix[b+1]
        long long lo_b = 0, hi_b = p.nb;
        while (hi_b - lo_b > 1) {
            long long mid = (lo_b + hi_b) >> 1;
            if (p.seg_prefix[mid] <= t) lo_b = mid; else hi_b = mid;
        }
        const long long b = lo_b;
        const long long delta0 = p.delta_lo + b * NC;
        const long long delta1 = min(delta0 + NC - 1, p.delta_hi);
        const long long rlo = max(0ll, -delta1), rhi = min(n, n - max(delta0, 0ll));
        const long long q = rlo / H + (t - p.seg_prefix[b]);
        const long long r0 = max(q * H, rlo), r1 = min((q + 1) * H, rhi);

        // lane's diagonal and its valid row range inside the tile
        const long long delta = delta0 + cell;
        long long lo = max(r0, max(0ll, -delta));
        long long hi = min(r1, n - max(delta, 0ll));
        if (delta > p.delta_hi) hi = lo;

        // seeds: direct centred dot products at row lo (reading G8)
        T QT[DL];
#pragma unroll
        for (int kk = 0; kk < DL; ++kk) {
            const int dim = kk * G + g;
            T acc = (T)0;
            if (dim >= d) {
                acc = (T)-1;
            } else if (lo < hi) {
                const T* xq = tw_q + (long long)dim * L + lo;
                const T* xr = tw_r + (long long)dim * L + lo + delta;
                const T mq = mu_q[(long long)dim * n + lo], mr = mu_r[(long long)dim * n + lo + delta];
                for (int tt = 0; tt < m; ++tt) acc = fma(xq[tt] - mq, xr[tt] - mr, acc);
            }
            QT[kk] = acc;
        }

        const int s_end = (int)(r1 - r0) + CA * (RA - 1);
        const long long c0 = r0 + delta0;  // column of cell c = 0 at step 0
        for (int cc = 0; cc < CA - 1; ++cc) enter(false, c0 + cc, st_r);

        for (int s = 0; s < s_end; ++s) {
            __syncwarp();
            if (s >= 1) leave(false, c0 + s - 1);
            if (s - 1 - CA * (RA - 1) >= 0) leave(true, r0 + s - 1 - CA * (RA - 1));
            if (s < r1 - r0) enter(true, r0 + s, st_q);
            enter(false, c0 + s + CA - 1, st_r);
            __syncwarp();

            const long long row = r0 + s - CA * a;
            const long long col = row + delta;
            const bool active = row >= lo && row < hi;
            const bool upd = row > lo && row < hi;
            const int sr = Gm::srow(row), sc = Gm::scol(col);

            // thresholds stay in registers for small per-lane dim counts; wide lanes
            // re-read them from the ring after the sort (register budget)
            constexpr bool KEEP = (DL <= 16 && G == 1);
            T S[DL], tr[KEEP ? DL : 1], tc[KEEP ? DL : 1];
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) {
                const int pl = kk * G + g;
                const V4 R = rowv[pl * PSR + sr];
                const V4 C = colv[pl * PSC + sc];
                if (upd) QT[kk] = fma(R.x, C.y, fma(C.x, R.y, QT[kk]));   // Eq. (1) recurrence
                const T aa = R.z * C.z;
                S[kk] = PT<T>::sqrt_abs(fma(-QT[kk], aa, two_m));            // Eq. (1) distance
                if constexpr (KEEP) {
                    tr[kk] = R.w;
                    tc[kk] = C.w;
                }
            }
            sort_net<T, DL>(S);                                              // Eq. (2) sort
            if (G > 1) lane_merge<T, DL, G>(S, g);
#pragma unroll
            for (int kk = 1; kk < DL; ++kk) S[kk] += S[kk - 1];              // Eq. (2) scan
            if (G > 1) {
                T tot = S[DL - 1];
#pragma unroll
                for (int dd = 1; dd < G; dd <<= 1) {
                    T y = __shfl_up_sync(FULL, tot, dd, G);
                    if (g >= dd) tot += y;
                }
                T excl = __shfl_up_sync(FULL, tot, 1, G);
                if (g == 0) excl = (T)0;
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) S[kk] += excl;
            }
            bool hit = false;
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) {
                const int pl = kk * G + g;
                if constexpr (KEEP) {
                    hit |= S[kk] <= tr[kk];
                    if (SELF) hit |= S[kk] <= tc[kk];
                } else {
                    hit |= S[kk] <= rowv[pl * PSR + sr].w;
                    if (SELF) hit |= S[kk] <= colv[pl * PSC + sc].w;
                }
            }
            hit = hit && active;
            if (__any_sync(FULL, hit)) {
                // Eq. (3) with the lowest-index tie rule: group min by shuffles, one leader
                // per row / column group compares (value, index) with the ring's best.
#pragma unroll
                for (int kk = 0; kk < DL; ++kk) ssc[kk * 32 + lane] = active ? S[kk] : INF;
                __syncwarp();
#pragma unroll 1
                for (int kk = 0; kk < DL; ++kk) {
                    const int pl = kk * G + g;
                    const T v = ssc[kk * 32 + lane];
                    T vr = v;
#pragma unroll
                    for (int bit = 0; bit < Gm::LOG_CA; ++bit)
                        vr = PT<T>::vmin(vr, __shfl_xor_sync(FULL, vr, 1 << (bit + Gm::LOG_G)));
                    const unsigned eqr = __ballot_sync(FULL, v == vr) & gmask_row;
                    if (vr < INF && lane == __ffs(eqr) - 1) {
                        const int ix = pl * PSR + sr;
                        const T cur = rowv[ix].w;
                        const unsigned ci = rowi[ix] & ~DIRTY;
                        if (vr < cur || (vr == cur && (unsigned)col < ci)) {
                            rowv[ix].w = vr;
                            rowi[ix] = (unsigned)col | DIRTY;
                        }
                    }
                    if (SELF) {
                        T vc = v;
#pragma unroll
                        for (int bit = 0; bit < 5 - Gm::LOG_G - Gm::LOG_CA; ++bit)
                            vc = PT<T>::vmin(vc, __shfl_xor_sync(FULL, vc, 1 << (bit + Gm::LOG_G + Gm::LOG_CA)));
                        const unsigned eqc = __ballot_sync(FULL, v == vc) & gmask_col;
                        // lowest row index = highest a = highest lane
                        if (vc < INF && eqc != 0 && lane == 31 - __clz(eqc)) {
                            const int ix = pl * PSC + sc;
                            const T cur = colv[ix].w;
                            const unsigned ci = coli[ix] & ~DIRTY;
                            if (vc < cur || (vc == cur && (unsigned)row < ci)) {
                                colv[ix].w = vc;
                                coli[ix] = (unsigned)row | DIRTY;
                            }
                        }
                    }
                }
            }
        }
        __syncwarp();
        // epilogue: the last row and the last CA columns are still in the rings
        if (r1 - r0 >= 1) leave(true, r1 - 1);
        for (int v = s_end - 1; v <= s_end + CA - 2; ++v) leave(false, c0 + v);
        __syncwarp();
    }
}


template <class T, int DL, int G, bool SELF> struct Inst {
    static size_t smem();
    static cudaError_t launch(const MainParams& p, int grid, cudaStream_t s);
    static int blocks_per_sm();
};

#ifdef MP_DIAG_IMPL
template <class T, int DL, int G, bool SELF> size_t Inst<T, DL, G, SELF>::smem() {
    return Smem<T, DL, G>::bytes_per_warp * WARPS_PER_BLOCK;
}
template <class T, int DL, int G, bool SELF>
cudaError_t Inst<T, DL, G, SELF>::launch(const MainParams& p, int grid, cudaStream_t s) {
    const size_t sm = smem();
    cudaError_t e = cudaFuncSetAttribute(mp_diag<T, DL, G, SELF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    mp_diag<T, DL, G, SELF><<<grid, WARPS_PER_BLOCK * 32, sm, s>>>(p);
    return cudaGetLastError();
}
template <class T, int DL, int G, bool SELF> int Inst<T, DL, G, SELF>::blocks_per_sm() {
    const size_t sm = smem();
    cudaFuncSetAttribute(mp_diag<T, DL, G, SELF>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    int nb = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, mp_diag<T, DL, G, SELF>, WARPS_PER_BLOCK * 32, sm);
    return nb;
}
#endif



}  // namespace mpk

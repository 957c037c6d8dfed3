// mp_kernels.cu -- precompute, key and finalize kernels + dispatch of the fused kernel.
// The fused diagonal kernel itself lives in mp_diag.cuh (instantiated in inst_*.cu so
// the heavy template variants compile in parallel).
#include "mp_diag16.cuh"
#include "mp_diag64f.cuh"
#include "mp_diag_cta.cuh"
#include "mp_diag_cta16.cuh"
#include "mp_diag_cta64.cuh"
#include "mp_diag_ctab.cuh"

#ifndef MP_MIX_STATS_KAHAN
#define MP_MIX_STATS_KAHAN 0   // Mixed window statistics with Kahan sums (1: experiment; FP16CK has them)
#endif

namespace mpk {

// ------------------------------------------------------------------ precompute
// Per window (dim, pos): two-pass mean and norm in the precalc precision (Fig. 1 table,
// L420-444), then df / dg (reading G7) and a = sqrt(2m)/norm (0 for flat windows, G4).
template <class T>
__global__ void pre_stats(const PreParams p) {
    const int d = p.d, m = p.m;
    const long long cntp = p.s_end - p.s_off;   // scratch window [s_off, s_end)
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (gid >= cntp * d) return;
    const int dim = (int)(gid / cntp);
    const long long pos = p.s_off + gid % cntp;
    const long long so = (long long)dim * p.s_ld + (pos - p.s_off);
    const double* x = p.T + (long long)dim * p.T_ld + (pos - p.T_off);
    // two-pass with compensated (Kahan) sums in the precalc precision; the paper leaves the
    // precalculation formulas out and stresses its accuracy (L792-794)
    T s = 0, c = 0;
    for (int t = 0; t < m; ++t) {
        const T y = (T)x[t] - c;
        const T tt = s + y;
        c = (tt - s) - y;
        s = tt;
    }
    const T mu = s / (T)m;
    T q = 0;
    c = 0;
    for (int t = 0; t < m; ++t) {
        const T cx = (T)x[t] - mu;
        const T y = cx * cx - c;
        const T tt = q + y;
        c = (tt - q) - y;
        q = tt;
    }
    reinterpret_cast<T*>(p.mu)[so] = mu;
    const T nr = sqrt(q);
    if constexpr (sizeof(T) == 4) p.nrm32[so] = nr; else p.nrm64[so] = nr;
}

template <class T, class A = T>  // A: precalc arithmetic (FP32 mode: FP64, reading R1)
__global__ void pre_diff(const PreParams p) {
    using V4 = typename PT<T>::V4;
    const int d = p.d, m = p.m;
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (gid >= (p.w1 - p.w0) * d) return;
    const long long pos = p.w0 + gid / d;  // position-major output
    const int dim = (int)(gid % d);
    const double* x = p.T + (long long)dim * p.T_ld - p.T_off;                    // x[t]
    const A* mu = reinterpret_cast<const A*>(p.mu) + (long long)dim * p.s_ld - p.s_off;  // mu[pos]
    const long long so = (long long)dim * p.s_ld + (pos - p.s_off);
    A nr;
    if constexpr (sizeof(A) == 4) nr = p.nrm32[so]; else nr = p.nrm64[so];
    V4 v;
    if (pos == 0) {
        v.x = 0; v.y = 0;
    } else {
        const A xl = (A)x[pos + m - 1], xf = (A)x[pos - 1];
        v.x = (T)((xl - xf) / (A)2);
        v.y = (T)((xl - mu[pos]) + (xf - mu[pos - 1]));
    }
    v.z = nr > (A)0 ? (T)(sqrt((A)(2 * m)) / nr) : (T)0;
    v.w = 0;
    reinterpret_cast<V4*>(p.st)[pos * d + dim] = v;
}

// position-major, zero-padded copies of the working-precision series and window means
// (the seeds' operands: a lane's dims are contiguous, so they load as vectors)
template <class T, class A = T>
__global__ void pre_pm(const PreParams p) {
    const int d = p.d, Dp = p.Dp;
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (gid >= (p.w1 + p.m - 1 - p.w0) * Dp) return;
    const long long t = p.w0 + gid / Dp;
    const int dim = (int)(gid % Dp);
    T* tw = reinterpret_cast<T*>(p.tw);
    T* mup = reinterpret_cast<T*>(p.mup);
    // pm_G > 0: dim kk*G + g is stored at g*DL + kk (each lane's dims contiguous)
    const long long o = p.pm_G > 0 ? t * Dp + (dim % p.pm_G) * p.pm_DL + dim / p.pm_G : t * Dp + dim;
    tw[o] = dim < d ? (T)p.T[(long long)dim * p.T_ld + (t - p.T_off)] : (T)0;
    if (t < p.w1) mup[o] = dim < d ? (T)reinterpret_cast<const A*>(p.mu)[(long long)dim * p.s_ld + (t - p.s_off)] : (T)0;
}

// ------------------------------------------------------------------ precompute, FP16 / Mixed
// Reading G16: an exact power-of-two scale s_k per dimension keeps the half-precision
// window energies (QT, norm^2) <= 2^14 (and, for FP16, the window sums <= 2^14); z-normalised
// distances are invariant under it (pinned in tests/test_oracle.py).
__global__ void pre_scale_max(const PreParams p) {
    const int d = p.d, m = p.m;
    const long long cntp = p.w1 - p.w0;
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (gid >= cntp * d) return;
    const int dim = (int)(gid / cntp);
    const long long pos = p.w0 + gid % cntp;
    const double* x = p.T + (long long)dim * p.T_ld + (pos - p.T_off);
    double s = 0, amax = 0;
    for (int t = 0; t < m; ++t) { s += x[t]; amax = fmax(amax, fabs(x[t])); }
    const double mu = s / m;
    double q = 0;
    for (int t = 0; t < m; ++t) q = fma(x[t] - mu, x[t] - mu, q);
    atomicMax(&p.maxbits[dim], (unsigned long long)__double_as_longlong(sqrt(q)));
    atomicMax(&p.maxbits[d + dim], (unsigned long long)__double_as_longlong(amax));
}
__global__ void pre_scale_pick(const PreParams p, int pure16) {
    const int dim = blockIdx.x * blockDim.x + threadIdx.x;
    if (dim >= p.d) return;
    const double nmax = __longlong_as_double((long long)p.maxbits[dim]);
    const double amax = __longlong_as_double((long long)p.maxbits[p.d + dim]);
    int e = 0;
    if (nmax > 0) e = (int)floor(log2(128.0 / nmax));
    if (pure16 && amax > 0) e = min(e, (int)floor(log2(16384.0 / ((double)p.m * amax))));
    e = max(-60, min(60, e));
    p.scale[dim] = ldexp(1.0, e);
}
// T = float: Mixed (plain FP32 sums, L777-785) or FP16CK (KAHAN: FP32 with Kahan-compensated
// sums, the text's FP16C reading L786-791); T = __half: FP16 or FP16C (KAHAN, Fig. 1 reading)
template <class T, bool KAHAN = false>
__global__ void pre_stats_h(const PreParams p) {
    const int d = p.d, m = p.m;
    const long long cntp = p.s_end - p.s_off;   // scratch window [s_off, s_end)
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (gid >= cntp * d) return;
    const int dim = (int)(gid / cntp);
    const long long pos = p.s_off + gid % cntp;
    const double sc = p.scale[dim];
    const double* x = p.T + (long long)dim * p.T_ld + (pos - p.T_off);
    T mu, nr;
    if constexpr (sizeof(T) == 4 && KAHAN) {  // FP16CK: FP32 two-pass, Kahan-compensated sums
        float s = 0, c = 0;
        for (int t = 0; t < m; ++t) { const float y = (float)(sc * x[t]) - c; const float tt = s + y; c = (tt - s) - y; s = tt; }
        mu = s / (float)m;
        float q = 0;
        c = 0;
        for (int t = 0; t < m; ++t) {
            const float cx = (float)(sc * x[t]) - mu;
            const float y = cx * cx - c; const float tt = q + y; c = (tt - q) - y; q = tt;
        }
        nr = sqrtf(q);
    } else if constexpr (sizeof(T) == 4) {  // Mixed: FP32 two-pass, plain sums
        float s = 0;
        for (int t = 0; t < m; ++t) s += (float)(sc * x[t]);
        mu = s / (float)m;
        float q = 0;
        for (int t = 0; t < m; ++t) {
            const float cx = (float)(sc * x[t]) - mu;
            q = fmaf(cx, cx, q);
        }
        nr = sqrtf(q);
    } else if constexpr (!KAHAN) {  // FP16 mode: plain half arithmetic (the paper's FP16 precalc)
        __half s = __float2half(0.f);
        for (int t = 0; t < m; ++t) s = __hadd(s, __double2half(sc * x[t]));
        mu = __hdiv(s, __int2half_rn(m));
        __half q = __float2half(0.f);
        for (int t = 0; t < m; ++t) {
            const __half cx = __hsub(__double2half(sc * x[t]), mu);
            q = __hfma(cx, cx, q);
        }
        nr = hsqrt(q);
    } else {  // FP16C: half arithmetic with Kahan-compensated sums (Fig. 1 "FP16 with compensator")
        __half s = __float2half(0.f), c = __float2half(0.f);
        for (int t = 0; t < m; ++t) {
            const __half y = __hsub(__double2half(sc * x[t]), c);
            const __half tt = __hadd(s, y);
            c = __hsub(__hsub(tt, s), y);
            s = tt;
        }
        mu = __hdiv(s, __int2half_rn(m));
        __half q = __float2half(0.f);
        c = __float2half(0.f);
        for (int t = 0; t < m; ++t) {
            const __half cx = __hsub(__double2half(sc * x[t]), mu);
            const __half y = __hsub(__hmul(cx, cx), c);
            const __half tt = __hadd(q, y);
            c = __hsub(__hsub(tt, q), y);
            q = tt;
        }
        nr = hsqrt(q);
    }
    reinterpret_cast<T*>(p.mu)[(long long)dim * p.s_ld + (pos - p.s_off)] = mu;
    reinterpret_cast<T*>(p.nrm32)[(long long)dim * p.s_ld + (pos - p.s_off)] = nr;   // typed scratch
}
template <class T>
__global__ void pre_diff_h(const PreParams p) {
    const int d = p.d, m = p.m;
    const long long f0 = p.w0 > 0 ? p.w0 - 1 : 0;   // flat scratch for [f0, s_end) (pre_fmt_h)
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (gid >= (p.s_end - f0) * d) return;
    const long long pos = f0 + gid / d;
    const int dim = (int)(gid % d);
    const double sc = p.scale[dim];
    const double* x = p.T + (long long)dim * p.T_ld - p.T_off;                       // x[t]
    const T* mu = reinterpret_cast<const T*>(p.mu) + (long long)dim * p.s_ld - p.s_off;  // mu[pos]
    const T nr = reinterpret_cast<const T*>(p.nrm32)[(long long)dim * p.s_ld + (pos - p.s_off)];
    __half* flat = reinterpret_cast<__half*>(p.flat);
    float df = 0, dg = 0, av;
    if constexpr (sizeof(T) == 4) {
        if (pos > 0) {
            const float xl = (float)(sc * x[pos + m - 1]), xf = (float)(sc * x[pos - 1]);
            df = (xl - xf) / 2.f;
            dg = (xl - mu[pos]) + (xf - mu[pos - 1]);
        }
        av = nr > 0.f ? sqrtf((float)(2 * m)) / nr : 0.f;
    } else {
        if (pos > 0) {
            const __half xl = __double2half(sc * x[pos + m - 1]), xf = __double2half(sc * x[pos - 1]);
            df = __half2float(__hdiv(__hsub(xl, xf), __float2half(2.f)));
            dg = __half2float(__hadd(__hsub(xl, mu[pos]), __hsub(xf, mu[pos - 1])));
        }
        av = __half2float(nr) > 0.f ? __half2float(__hdiv(hsqrt(__int2half_rn(2 * m)), nr)) : 0.f;
    }
    av = fminf(av, 65504.f);  // finite half (near-flat windows)
    const long long o = (pos - p.s_off) * d + dim, nd = p.s_ld * d;
    flat[o] = __float2half_rn(df);
    flat[nd + o] = __float2half_rn(dg);
    flat[2 * nd + o] = __float2half_rn(av);
}
// row format (x, x) and pair format (x_pos, x_pos+1) H4 entries for the half2 kernel.  The
// pair array has n+1 entries: entry e holds (x_{e-1}, x_e), so a pair starting at column -1
// (an AB-join diagonal start) still finds its second cell's data.
__global__ void pre_fmt_h(const PreParams p) {
    const long long n = p.n;
    const int d = p.d;
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (gid >= (p.w1 - p.w0 + 1) * d) return;   // pair entries [w0, w1]
    const long long e = p.w0 + gid / d;          // pair entry; first position e - 1
    const int dim = (int)(gid % d);
    const __half* f = reinterpret_cast<const __half*>(p.flat);
    const long long nd = p.s_ld * d;
    const __half z = __float2half(0.f);
    const long long ia = (e - 1 - p.s_off) * d + dim, ib = (e - p.s_off) * d + dim;
    const bool va = e >= 1, vb = e < n;
    H4 q;
    q.x = __halves2half2(va ? f[ia] : z, vb ? f[ib] : z);
    q.y = __halves2half2(va ? f[nd + ia] : z, vb ? f[nd + ib] : z);
    q.z = __halves2half2(va ? f[2 * nd + ia] : z, vb ? f[2 * nd + ib] : z);
    q.w = __half2half2(z);
    reinterpret_cast<H4*>(p.st_pair)[e * d + dim] = q;
    if (vb && e < p.w1) {  // row format: one position (the kernel broadcasts it to both cells of a pair)
        RH r;
        r.df = f[ib]; r.dg = f[nd + ib]; r.a = f[2 * nd + ib]; r.t = z;
        reinterpret_cast<RH*>(p.st)[e * d + dim] = r;
    }
}
template <class T>
__global__ void pre_pm_h(const PreParams p) {
    const int d = p.d, Dp = p.Dp;
    const long long gid0 = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (gid0 >= (p.w1 + p.m - 1 - p.w0) * Dp) return;
    const long long gid = p.w0 * Dp + gid0;       // absolute [t][Dp] index
    const long long t = gid / Dp;
    const int dim = (int)(gid % Dp);
    T* tw = reinterpret_cast<T*>(p.tw);
    T* mup = reinterpret_cast<T*>(p.mup);
    if (dim < d) {
        const double v = p.scale[dim] * p.T[(long long)dim * p.T_ld + (t - p.T_off)];
        if constexpr (sizeof(T) == 4) tw[gid] = (float)v; else tw[gid] = __double2half(v);
    } else {
        tw[gid] = (T)0.f;
    }
    if (t < p.w1) mup[gid] = dim < d ? reinterpret_cast<const T*>(p.mu)[(long long)dim * p.s_ld + (t - p.s_off)] : (T)0.f;
}

// ------------------------------------------------------------------ keys
__global__ void init_keys32(unsigned long long* k, long long count) {
    const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < count) k[i] = EMPTY32;
}
__global__ void init_keys64(K64* k, long long count) {
    const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < count) { k[i].v = EMPTY64V; k[i].i = EMPTY64I; }
}
// FP64 AoS keys -> two int64 planes (value bits, index) for the collective merge
__global__ void keys64_to_ext(const K64* k, long long* ext, long long count) {
    const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < count) {
        ext[i] = (long long)k[i].v;
        ext[count + i] = (k[i].v == EMPTY64V) ? EXT_EMPTY : (long long)k[i].i;
    }
}
__global__ void key_mask(long long count, long long* ext, const long long* gv) {
    const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < count && ext[i] != gv[i]) ext[count + i] = EXT_EMPTY;
}
// ext keys [pos][rank] -> P [rank][pos] (sum / (k+1), reading G11), I [rank][pos]
__global__ void finalize32(const unsigned long long* k, long long n, int d, double* P, long long* I) {
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (gid >= n * d) return;
    const long long pos = gid / d;
    const int rk = (int)(gid % d);
    const unsigned long long key = k[gid];
    double pv;
    long long ix;
    if (key >= EMPTY32) { pv = __longlong_as_double(0x7ff0000000000000ll); ix = -1; }
    else { pv = (double)__uint_as_float((unsigned)(key >> 32)) / (double)(rk + 1); ix = (long long)(unsigned)key; }
    P[(long long)rk * n + pos] = pv;
    I[(long long)rk * n + pos] = ix;
}
__global__ void finalize64(const long long* ext, long long n, int d, double* P, long long* I) {
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const long long count = n * d;
    if (gid >= count) return;
    const long long pos = gid / d;
    const int rk = (int)(gid % d);
    const unsigned long long v = (unsigned long long)ext[gid];
    const long long ix = ext[count + gid];
    double pv;
    long long oi;
    if (v >= EMPTY64V || ix == EXT_EMPTY) { pv = __longlong_as_double(0x7ff0000000000000ll); oi = -1; }
    else { pv = __longlong_as_double((long long)v) / (double)(rk + 1); oi = ix; }
    P[(long long)rk * n + pos] = pv;
    I[(long long)rk * n + pos] = oi;
}
// streamed finalize (mp_compute_stream): internal keys of positions [p0, p1) -> window buffers
// P, I [rank][p1 - p0]; same arithmetic as finalize32 / keys64_to_ext + finalize64
__global__ void finalize_window32(const unsigned long long* k, long long p0, long long p1, int d, double* P, long long* I) {
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const long long w = p1 - p0;
    if (gid >= w * d) return;
    const long long pos = p0 + gid / d;
    const int rk = (int)(gid % d);
    const unsigned long long key = k[pos * d + rk];
    double pv;
    long long ix;
    if (key >= EMPTY32) { pv = __longlong_as_double(0x7ff0000000000000ll); ix = -1; }
    else { pv = (double)__uint_as_float((unsigned)(key >> 32)) / (double)(rk + 1); ix = (long long)(unsigned)key; }
    P[(long long)rk * w + (pos - p0)] = pv;
    I[(long long)rk * w + (pos - p0)] = ix;
}
__global__ void finalize_window64(const K64* k, long long p0, long long p1, int d, double* P, long long* I) {
    const long long gid = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    const long long w = p1 - p0;
    if (gid >= w * d) return;
    const long long pos = p0 + gid / d;
    const int rk = (int)(gid % d);
    const K64 key = k[pos * d + rk];
    double pv;
    long long oi;
    if (key.v >= EMPTY64V) { pv = __longlong_as_double(0x7ff0000000000000ll); oi = -1; }
    else { pv = __longlong_as_double((long long)key.v) / (double)(rk + 1); oi = (long long)key.i; }
    P[(long long)rk * w + (pos - p0)] = pv;
    I[(long long)rk * w + (pos - p0)] = oi;
}
__global__ void check_finite(const double* x, long long count, int* flag) {
    for (long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x; i < count;
         i += (long long)gridDim.x * blockDim.x)
        if (!isfinite(x[i])) atomicOr(flag, 1);
}

// ------------------------------------------------------------------ dispatch
static inline unsigned grid1d(long long count, int bs) { return (unsigned)((count + bs - 1) / bs); }

Variant pick_variant(int prec, int d) {
    // A lane holds DL <= 16 dims (register budget; DL = 32 only for FP32 d > 512); for small
    // d a lane owns W = 2 adjacent diagonals (d <= 8).
    if (prec == P16CK) prec = PMIX;   // same kernels as Mixed
    if (prec == P32N) prec = P32;     // same shapes as FP32
    int dp = 1;
    while (dp < d) dp <<= 1;
    Variant v;
    if (prec == P16 || prec == PMIX || prec == P16C) {  // half2: a lane-cell is a pair of diagonals
        if (dp <= 16) { v.DL = dp; v.G = 1; }
        else if (dp <= 256) { v.DL = 8; v.G = dp / 8; if (MP_CTAH_NW && dp >= MP_CTAH_MIN_DP) v.cta = v.G == 16 ? CtaShapeH<16>::NW : v.G == 8 ? CtaShapeH<8>::NW : CtaShapeH<32>::NW; }
        else { v.DL = dp / 32; v.G = 32; }
        v.W = 2;
    } else if (prec == P64) {  // FP64 with the FP32 filter (mp_diag64f): one cell per lane-cell
        if (dp <= 16) { v.DL = dp; v.G = 1; v.W = 1; }
        else {
            v.DL = 16; v.G = dp / 16; v.W = 1;
            if (MP_CTA64_ON && dp >= MP_CTA64_MIN_DP && dp / MP_CTA64_DL <= 32) {
                v.DL = MP_CTA64_DL;
                v.G = dp / v.DL;
                v.cta = v.G == 4 ? CtaShape64<4>::NW : v.G == 8 ? CtaShape64<8>::NW : v.G == 16 ? CtaShape64<16>::NW : CtaShape64<32>::NW;
            }
        }
    } else {
        if (dp <= 8) { v.DL = dp; v.G = 1; v.W = 2; }
        else if (dp == 16) { v.DL = 16; v.G = 1; v.W = 1; if (MP_CTA_NW && dp >= MP_CTA_MIN_DP) v.cta = MP_CTA_NW; }
        else if (MP_CTAB_ON && dp >= 64) { v.DL = ctab_dl(dp); v.G = dp / v.DL; v.W = 1; v.cta = MP_CTAB_NT / 32; v.ctab = true; }
        else if (dp <= 512) { v.DL = 16; v.G = dp / 16; v.W = 1; if (MP_CTA_NW && dp >= MP_CTA_MIN_DP) v.cta = MP_CTA_NW; }
        else { v.DL = 32; v.G = dp / 32; v.W = 1; }
    }
    v.NC = v.cta ? 32 * v.cta / v.G * v.W : 32 / v.G * v.W;
    return v;
}

// op: 0 = smem, 1 = launch, 2 = blocks/SM, 3 = warps/block
template <class T, bool SELF, bool COMP = true>
static long long dispatch_t(int op, int DL, int G, int W, const MainParams* p, int grid, cudaStream_t s) {
#define MP_CASE(dl, g, w)                                                                  \
    if (DL == dl && G == g && W == w) {                                                    \
        if (op == 0) return (long long)Inst<T, dl, g, w, SELF, COMP>::smem();              \
        if (op == 1) return (long long)Inst<T, dl, g, w, SELF, COMP>::launch(*p, grid, s); \
        if (op == 3) return Inst<T, dl, g, w, SELF, COMP>::warps_per_block();              \
        return Inst<T, dl, g, w, SELF, COMP>::blocks_per_sm();                             \
    }
    if constexpr (sizeof(T) == 4) {
        MP_CASE(1, 1, 2) MP_CASE(2, 1, 2) MP_CASE(4, 1, 2) MP_CASE(8, 1, 2) MP_CASE(16, 1, 1)
        MP_CASE(16, 2, 1) MP_CASE(16, 4, 1) MP_CASE(16, 8, 1) MP_CASE(16, 16, 1) MP_CASE(16, 32, 1) MP_CASE(32, 32, 1)
    }
#undef MP_CASE
    return op == 1 ? (long long)cudaErrorInvalidValue : 0;
}

template <bool SELF, int MIXED>
static long long dispatch_h(int op, int DL, int G, const MainParams* p, int grid, cudaStream_t s) {
#define MP_HCASE(dl, g)                                                                    \
    if (DL == dl && G == g) {                                                              \
        if (op == 0) return (long long)InstH<dl, g, SELF, MIXED>::smem();                  \
        if (op == 1) return (long long)InstH<dl, g, SELF, MIXED>::launch(*p, grid, s);     \
        if (op == 3) return InstH<dl, g, SELF, MIXED>::warps_per_block();                  \
        return InstH<dl, g, SELF, MIXED>::blocks_per_sm();                                 \
    }
    MP_HCASE(1, 1) MP_HCASE(2, 1) MP_HCASE(4, 1) MP_HCASE(8, 1) MP_HCASE(16, 1)
    MP_HCASE(8, 2) MP_HCASE(8, 4) MP_HCASE(8, 8) MP_HCASE(8, 16) MP_HCASE(8, 32) MP_HCASE(16, 32) MP_HCASE(32, 32)
#undef MP_HCASE
    return op == 1 ? (long long)cudaErrorInvalidValue : 0;
}

template <bool SELF>
static long long dispatch_64f(int op, int DL, int G, const MainParams* p, int grid, cudaStream_t s) {
#define MP_FCASE(dl, g)                                                                    \
    if (DL == dl && G == g) {                                                              \
        if (op == 0) return (long long)Inst64F<dl, g, SELF>::smem();                       \
        if (op == 1) return (long long)Inst64F<dl, g, SELF>::launch(*p, grid, s);          \
        if (op == 3) return Inst64F<dl, g, SELF>::warps_per_block();                       \
        return Inst64F<dl, g, SELF>::blocks_per_sm();                                      \
    }
    MP_FCASE(1, 1) MP_FCASE(2, 1) MP_FCASE(4, 1) MP_FCASE(8, 1) MP_FCASE(16, 1)
    MP_FCASE(16, 2) MP_FCASE(16, 4) MP_FCASE(16, 8) MP_FCASE(16, 16) MP_FCASE(16, 32)
#undef MP_FCASE
    return op == 1 ? (long long)cudaErrorInvalidValue : 0;
}

template <bool SELF>
static long long dispatch_cta(int op, int G, const MainParams* p, int grid, cudaStream_t s) {
#define MP_CCASE(g)                                                                        \
    if (G == g) {                                                                          \
        using I = InstCta<16, g, MP_CTA_NW, SELF>;                                         \
        if (op == 0) return (long long)I::smem();                                          \
        if (op == 1) return (long long)I::launch(*p, grid, s);                             \
        if (op == 3) return 1;  /* one tile per block */                                   \
        return I::blocks_per_sm();                                                         \
    }
#if MP_CTA_NW
#if MP_CTA_MIN_DP < 64  // measured slower than the warp kernel at d = 16 (C2: 55.9 vs 40.6 ms)
    MP_CCASE(1) MP_CCASE(2)
#endif
    MP_CCASE(4) MP_CCASE(8) MP_CCASE(16) MP_CCASE(32)
#endif
#undef MP_CCASE
    return op == 1 ? (long long)cudaErrorInvalidValue : 0;
}

template <bool SELF>
static long long dispatch_ctab(int op, int dpad, const MainParams* p, int grid, cudaStream_t s) {
#define MP_BCASE(dp)                                                                       \
    if (dpad == dp) {                                                                      \
        using I = InstCtab<ctab_dl(dp), dp / ctab_dl(dp), MP_CTAB_NT, SELF>;               \
        if (op == 0) return (long long)I::smem();                                          \
        if (op == 1) return (long long)I::launch(*p, grid, s);                             \
        if (op == 3) return 1;  /* one tile per block */                                   \
        return I::blocks_per_sm();                                                         \
    }
#if MP_CTAB_ON
    MP_BCASE(64) MP_BCASE(128) MP_BCASE(256) MP_BCASE(512) MP_BCASE(1024)
#endif
#undef MP_BCASE
    return op == 1 ? (long long)cudaErrorInvalidValue : 0;
}

template <bool SELF, int MODE>
static long long dispatch_ctah(int op, int G, const MainParams* p, int grid, cudaStream_t s) {
#define MP_HCCASE(g)                                                                       \
    if (G == g) {                                                                          \
        using I = InstCtaH<8, g, CtaShapeH<g>::NW, SELF, MODE>;                                  \
        if (op == 0) return (long long)I::smem();                                          \
        if (op == 1) return (long long)I::launch(*p, grid, s);                             \
        if (op == 3) return 1;  /* one tile per block */                                   \
        return I::blocks_per_sm();                                                         \
    }
#if MP_CTAH_NW
    MP_HCCASE(8) MP_HCCASE(16) MP_HCCASE(32)
#endif
#undef MP_HCCASE
    return op == 1 ? (long long)cudaErrorInvalidValue : 0;
}

template <bool SELF>
static long long dispatch_cta64(int op, int G, const MainParams* p, int grid, cudaStream_t s) {
#define MP_DCCASE(g)                                                                       \
    if (G == g) {                                                                          \
        using I = InstCta64<MP_CTA64_DL, g, CtaShape64<g>::NW, SELF>;                      \
        if (op == 0) return (long long)I::smem();                                          \
        if (op == 1) return (long long)I::launch(*p, grid, s);                             \
        if (op == 3) return 1;  /* one tile per block */                                   \
        return I::blocks_per_sm();                                                         \
    }
#if MP_CTA64_ON
    MP_DCCASE(4) MP_DCCASE(8) MP_DCCASE(16) MP_DCCASE(32)
#endif
#undef MP_DCCASE
    return op == 1 ? (long long)cudaErrorInvalidValue : 0;
}

static long long dispatch(int op, int prec, bool self, int d, const MainParams* p, int grid, cudaStream_t s) {
    const Variant v = pick_variant(prec, d);
    if (v.cta && (prec == P16 || prec == PMIX || prec == P16C || prec == P16CK)) {
        // half-kernel modes (mp_diag16.cuh): FP16CK = Mixed with compensated seeds (3); a launch
        // with a tensor-core seed table (MainParams::seed_tab) takes the table kernel (5)
        const bool tab = p && p->seed_tab && (prec == PMIX || prec == P16CK);
        const int md = tab ? 5 : prec == P16 ? 0 : prec == PMIX ? 1 : prec == P16C ? 2 : 3;
        if (md == 0) return self ? dispatch_ctah<true, 0>(op, v.G, p, grid, s) : dispatch_ctah<false, 0>(op, v.G, p, grid, s);
        if (md == 1) return self ? dispatch_ctah<true, 1>(op, v.G, p, grid, s) : dispatch_ctah<false, 1>(op, v.G, p, grid, s);
        if (md == 2) return self ? dispatch_ctah<true, 2>(op, v.G, p, grid, s) : dispatch_ctah<false, 2>(op, v.G, p, grid, s);
        if (md == 3) return self ? dispatch_ctah<true, 3>(op, v.G, p, grid, s) : dispatch_ctah<false, 3>(op, v.G, p, grid, s);
        return self ? dispatch_ctah<true, 5>(op, v.G, p, grid, s) : dispatch_ctah<false, 5>(op, v.G, p, grid, s);
    }
    if (v.cta && prec == P64) return self ? dispatch_cta64<true>(op, v.G, p, grid, s) : dispatch_cta64<false>(op, v.G, p, grid, s);
    if (v.ctab) return self ? dispatch_ctab<true>(op, v.DL * v.G, p, grid, s) : dispatch_ctab<false>(op, v.DL * v.G, p, grid, s);
    if (v.cta) return self ? dispatch_cta<true>(op, v.G, p, grid, s) : dispatch_cta<false>(op, v.G, p, grid, s);
    if (prec == P16) return self ? dispatch_h<true, 0>(op, v.DL, v.G, p, grid, s) : dispatch_h<false, 0>(op, v.DL, v.G, p, grid, s);
    if (prec == PMIX) return self ? dispatch_h<true, 1>(op, v.DL, v.G, p, grid, s) : dispatch_h<false, 1>(op, v.DL, v.G, p, grid, s);
    if (prec == P16C) return self ? dispatch_h<true, 2>(op, v.DL, v.G, p, grid, s) : dispatch_h<false, 2>(op, v.DL, v.G, p, grid, s);
    if (prec == P16CK) return self ? dispatch_h<true, 3>(op, v.DL, v.G, p, grid, s) : dispatch_h<false, 3>(op, v.DL, v.G, p, grid, s);
    if (prec == P64) return self ? dispatch_64f<true>(op, v.DL, v.G, p, grid, s) : dispatch_64f<false>(op, v.DL, v.G, p, grid, s);
    if (prec == P32) return self ? dispatch_t<float, true>(op, v.DL, v.G, v.W, p, grid, s) : dispatch_t<float, false>(op, v.DL, v.G, v.W, p, grid, s);
    if (prec == P32N) return self ? dispatch_t<float, true, false>(op, v.DL, v.G, v.W, p, grid, s) : dispatch_t<float, false, false>(op, v.DL, v.G, v.W, p, grid, s);
    return op == 1 ? (long long)cudaErrorInvalidValue : 0;
}

int variant_warps_per_block(int prec, int d, bool self) { return (int)dispatch(3, prec, self, d, nullptr, 0, 0); }
size_t smem_per_block(int prec, int d, bool self) { return (size_t)dispatch(0, prec, self, d, nullptr, 0, 0); }
int main_blocks_per_sm(int prec, int d, bool self) { return (int)dispatch(2, prec, self, d, nullptr, 0, 0); }
cudaError_t launch_main(int prec, bool self, const MainParams& p, int grid, cudaStream_t s) {
    return (cudaError_t)dispatch(1, prec, self, p.d, &p, grid, s);
}

cudaError_t launch_scale_max(const PreParams& p, bool reset, cudaStream_t s) {
    if (reset) cudaMemsetAsync(p.maxbits, 0, 2 * p.d * sizeof(unsigned long long), s);
    pre_scale_max<<<grid1d((p.w1 - p.w0) * p.d, 256), 256, 0, s>>>(p);
    return cudaGetLastError();
}
cudaError_t launch_scale_pick(int prec, const PreParams& p, cudaStream_t s) {
    pre_scale_pick<<<grid1d(p.d, 128), 128, 0, s>>>(p, (prec == PMIX || prec == P16CK) ? 0 : 1);
    return cudaGetLastError();
}

cudaError_t launch_precompute(int prec, const PreParams& p, cudaStream_t s, bool with_scale) {
    const long long cs = (p.s_end - p.s_off) * p.d;          // window statistics (scratch)
    const long long cw = (p.w1 - p.w0) * p.d;                // stats entries written
    const long long cpm = (p.w1 + p.m - 1 - p.w0) * p.Dp;    // seed operands written
    if (prec == P64) {
        pre_stats<double><<<grid1d(cs, 256), 256, 0, s>>>(p);
        pre_diff<double><<<grid1d(cw, 256), 256, 0, s>>>(p);
        pre_pm<double><<<grid1d(cpm, 256), 256, 0, s>>>(p);
    } else if (prec == P32) {
        // FP32 mode: window stats and df / dg / a in FP64 from the FP64 input, rounded once to
        // FP32 (reading R1'): FP32 cancellation in x - mu grows with the window's offset.
        // (FP64 seeds from the FP64 series were measured too: no accuracy gain, C2 +11 %.)
        pre_stats<double><<<grid1d(cs, 256), 256, 0, s>>>(p);
        pre_diff<float, double><<<grid1d(cw, 256), 256, 0, s>>>(p);
        pre_pm<float, double><<<grid1d(cpm, 256), 256, 0, s>>>(p);
    } else {
        if (with_scale) {  // a streamed run computes the per-dimension scale over all windows first
            launch_scale_max(p, true, s);
            launch_scale_pick(prec, p, s);
        }
        const long long f0 = p.w0 > 0 ? p.w0 - 1 : 0;
        const long long cf = (p.s_end - f0) * p.d;          // flat scratch (pre_diff_h)
        if (prec == P16CK) {
            pre_stats_h<float, true><<<grid1d(cs, 256), 256, 0, s>>>(p);
            pre_diff_h<float><<<grid1d(cf, 256), 256, 0, s>>>(p);
            pre_pm_h<float><<<grid1d(cpm, 256), 256, 0, s>>>(p);
        } else if (prec == PMIX) {
            pre_stats_h<float, MP_MIX_STATS_KAHAN><<<grid1d(cs, 256), 256, 0, s>>>(p);
            pre_diff_h<float><<<grid1d(cf, 256), 256, 0, s>>>(p);
            pre_pm_h<float><<<grid1d(cpm, 256), 256, 0, s>>>(p);
        } else if (prec == P16C) {
            pre_stats_h<__half, true><<<grid1d(cs, 256), 256, 0, s>>>(p);
            pre_diff_h<__half><<<grid1d(cf, 256), 256, 0, s>>>(p);
            pre_pm_h<__half><<<grid1d(cpm, 256), 256, 0, s>>>(p);
        } else {
            pre_stats_h<__half><<<grid1d(cs, 256), 256, 0, s>>>(p);
            pre_diff_h<__half><<<grid1d(cf, 256), 256, 0, s>>>(p);
            pre_pm_h<__half><<<grid1d(cpm, 256), 256, 0, s>>>(p);
        }
        pre_fmt_h<<<grid1d((p.w1 - p.w0 + 1) * p.d, 256), 256, 0, s>>>(p);
    }
    return cudaGetLastError();
}

cudaError_t launch_init_keys(int prec, void* keys, long long count, cudaStream_t s) {
    if (prec == P64) init_keys64<<<grid1d(count, 256), 256, 0, s>>>(reinterpret_cast<K64*>(keys), count);
    else init_keys32<<<grid1d(count, 256), 256, 0, s>>>(reinterpret_cast<unsigned long long*>(keys), count);
    return cudaGetLastError();
}

cudaError_t launch_keys_to_ext(int prec, const void* keys, void* ext, long long count, cudaStream_t s) {
    if (prec == P64) {
        keys64_to_ext<<<grid1d(count, 256), 256, 0, s>>>(reinterpret_cast<const K64*>(keys), reinterpret_cast<long long*>(ext), count);
        return cudaGetLastError();
    }
    return cudaMemcpyAsync(ext, keys, count * sizeof(long long), cudaMemcpyDeviceToDevice, s);
}

cudaError_t launch_finalize_window(int prec, const void* keys, long long p0, long long p1, int d, double* P,
                                   long long* I, cudaStream_t s) {
    const long long cnt = (p1 - p0) * d;
    if (prec == P64) finalize_window64<<<grid1d(cnt, 256), 256, 0, s>>>(reinterpret_cast<const K64*>(keys), p0, p1, d, P, I);
    else finalize_window32<<<grid1d(cnt, 256), 256, 0, s>>>(reinterpret_cast<const unsigned long long*>(keys), p0, p1, d, P, I);
    return cudaGetLastError();
}

cudaError_t launch_key_mask(long long count, long long* ext, const long long* gv, cudaStream_t s) {
    key_mask<<<grid1d(count, 256), 256, 0, s>>>(count, ext, gv);
    return cudaGetLastError();
}

cudaError_t launch_finalize(int prec, const void* keys_ext, long long n, int d, double* P, long long* I, cudaStream_t s) {
    const long long cnt = n * d;
    if (prec == P64) finalize64<<<grid1d(cnt, 256), 256, 0, s>>>(reinterpret_cast<const long long*>(keys_ext), n, d, P, I);
    else finalize32<<<grid1d(cnt, 256), 256, 0, s>>>(reinterpret_cast<const unsigned long long*>(keys_ext), n, d, P, I);
    return cudaGetLastError();
}

// ------------------------------------------------------------------ stage self-tests
// One cell per G lanes, DL values per lane, exactly as the fused kernels hold them: lane g's
// register kk is dim kk G + g; the sort / merge / scan templates are the kernels' own.
template <int DL, int G, bool CTAB>
__global__ void selftest_sort_scan(int d, long long count, const float* in, float* out) {
    constexpr int CPW = 32 / G;  // cells per warp
    const long long cell = (blockIdx.x * (long long)blockDim.x + threadIdx.x) / G;
    const int g = threadIdx.x & (G - 1);
    const bool ok = cell < count;   // whole warps stay converged for the shuffles
    (void)CPW;
    float S[DL];
    // padded dims sort last (D ~ 1e18), or first with D = 0 in the sign-split merge (ranks shift)
    constexpr bool SIGN = CTAB && MP_CTAB_SIGN && G == 4;
#pragma unroll
    for (int kk = 0; kk < DL; ++kk) {
        const int dim = kk * G + g;
        S[kk] = (ok && dim < d) ? in[cell * d + dim] : (SIGN ? 0.f : PT<float>::pad_a());
    }
    if constexpr (G == 1 && DL >= 8 && last_layer_adjacent<DL>()) {
        sort_scan_fused<float, DL>(S);        // mp_diag, one lane per cell
    } else if constexpr (G == 1) {
        sort_net<float, DL>(S);
#pragma unroll
        for (int kk = 1; kk < DL; ++kk) S[kk] += S[kk - 1];
    } else {
        if constexpr (CTAB && MP_CTAB_SIGN && G == 4) {   // mp_diag_ctab, sign-split merge
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) S[kk] *= (g < 2 ? 1.f : -1.f);
            sort_net<float, DL>(S);
            sign_merge4<DL>(S, g);
            pair_scan<float, DL>(S);
            sign_offsets<DL>(S, g);
#pragma unroll
            for (int kk = 0; kk < DL; ++kk) {
                const int rk = sign_rank<DL>(g, kk) - (DL * G - d);
                if (ok && rk >= 0 && rk < d) out[cell * d + rk] = S[kk];
            }
            return;
        }
        sort_net<float, DL>(S);
        if constexpr (CTAB) {                 // mp_diag_ctab: last merge layer fused into the scan
            lane_merge<float, DL, G, true>(S, g);
            pair_scan<float, DL>(S);
        } else {                              // mp_diag, G lanes per cell: two half chains
            lane_merge<float, DL, G>(S, g);
#pragma unroll
            for (int kk = 1; kk < DL / 2; ++kk) S[kk] += S[kk - 1];
#pragma unroll
            for (int kk = DL / 2 + 1; kk < DL; ++kk) S[kk] += S[kk - 1];
#pragma unroll
            for (int kk = DL / 2; kk < DL; ++kk) S[kk] += S[DL / 2 - 1];
        }
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
#pragma unroll
    for (int kk = 0; kk < DL; ++kk) {
        const int rk = g * DL + kk;   // lane g holds ranks g DL .. g DL + DL - 1
        if (ok && rk < d) out[cell * d + rk] = S[kk];
    }
}

cudaError_t launch_selftest_sort_scan(int d, long long count, const float* in, float* out, cudaStream_t s) {
    const Variant v = pick_variant(P32, d);
    const long long threads = count * v.G;
    const unsigned grid = (unsigned)((threads + 127) / 128);
#define MP_STCASE(dl, g, ct)                                                                 \
    if (v.DL == dl && v.G == g && v.ctab == ct) {                                            \
        selftest_sort_scan<dl, g, ct><<<grid, 128, 0, s>>>(d, count, in, out);               \
        return cudaGetLastError();                                                           \
    }
    MP_STCASE(1, 1, false) MP_STCASE(2, 1, false) MP_STCASE(4, 1, false) MP_STCASE(8, 1, false)
    MP_STCASE(16, 1, false) MP_STCASE(16, 2, false) MP_STCASE(16, 4, true) MP_STCASE(16, 8, true)
    MP_STCASE(16, 16, true) MP_STCASE(16, 32, true) MP_STCASE(32, 32, true) MP_STCASE(32, 2, true)
    MP_STCASE(32, 4, true) MP_STCASE(32, 8, true) MP_STCASE(32, 16, true)
#undef MP_STCASE
    return cudaErrorInvalidValue;
}

template <class T>
__global__ void selftest_unpack(const typename PT<T>::V4* st, long long count, double* df, double* dg, double* a) {
    const long long i = blockIdx.x * (long long)blockDim.x + threadIdx.x;
    if (i < count) { df[i] = (double)st[i].x; dg[i] = (double)st[i].y; a[i] = (double)st[i].z; }
}
cudaError_t launch_selftest_unpack(int prec, const void* st, long long n, int d, double* df, double* dg, double* a,
                                   cudaStream_t s) {
    const long long cnt = n * d;
    if (prec == P64) selftest_unpack<double><<<grid1d(cnt, 256), 256, 0, s>>>(reinterpret_cast<const double4*>(st), cnt, df, dg, a);
    else if (prec == P32) selftest_unpack<float><<<grid1d(cnt, 256), 256, 0, s>>>(reinterpret_cast<const float4*>(st), cnt, df, dg, a);
    else return cudaErrorInvalidValue;
    return cudaGetLastError();
}

cudaError_t launch_check_finite(const double* x, long long count, int* flag, cudaStream_t s) {
    check_finite<<<1184, 256, 0, s>>>(x, count, flag);
    return cudaGetLastError();
}

}  // namespace mpk

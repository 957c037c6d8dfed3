// mp_seed_tc.cu -- QT seeds of the half-precision modes as a tensor-core GEMM (SURVEY 8(f)
// NEXT-3, the paper's future work "TF32 execution mode or BFLOAT16").
//
// A seed is the direct centred dot product QT(i0, j) = sum_t (x_q[i0+t] - mu_q[i0]) (x_r[j+t] - mu_r[j])
// (reading G8) at the re-seed rows i0 = r H.  For one dimension k the seeds of
// the rows r in [r_lo, r_hi) against the columns j in [j_lo, j_hi) form the matrix product
//     S_k = A_k B_k^T,  A_k[r][t] = x_q[rH + t] - mu_q[rH],  B_k[j][t] = x_r[j + t] - mu_r[j],
// with K = m: a dense contraction (B is a centred Hankel matrix).  One CTA computes a 128-row x
// 256-column tile for every dimension in turn: 128 threads build the K-chunks of A and B in
// shared memory (FP32 arithmetic of the Mixed precalc, rounded to FP16, UMMA K-major canonical
// layout without swizzle), one thread issues tcgen05.mma (kind::f16, FP32 accumulation in
// TMEM, M = 128, N = 256, K = 16 per instruction), the accumulator comes back with tcgen05.ld
// and is rounded to half -- the precision the half kernels hold QT in.  The operand chunks are
// double-buffered: building chunk c + 1 overlaps the MMAs of chunk c (tcgen05.commit ->
// mbarrier).
//
// Output: tab[((r - r_lo) * d + k) * ldj + (j - j_lo)] (half), ldj a multiple of 8.
#include "mp_internal.h"

#include <cuda_fp16.h>

namespace mpk {

namespace {

constexpr int TM = 128, TN = 256, KC = 64;      // tile rows / columns, K per operand chunk
constexpr int A_BYTES = TM * KC * 2, B_BYTES = TN * KC * 2;
constexpr int XS = TN + KC;                      // staged series values for one B chunk

__device__ __forceinline__ unsigned smem_addr(const void* p) { return (unsigned)__cvta_generic_to_shared(p); }

// UMMA shared-memory descriptor, K-major, no swizzle: core matrices of 8 rows x 16 bytes stored
// contiguously; SBO = byte distance between core matrices along M/N, LBO = along K.
__device__ __forceinline__ unsigned long long umma_desc(unsigned saddr, unsigned lbo, unsigned sbo) {
    unsigned long long d = 0;
    d |= (unsigned long long)((saddr >> 4) & 0x3FFF);
    d |= (unsigned long long)((lbo >> 4) & 0x3FFF) << 16;
    d |= (unsigned long long)((sbo >> 4) & 0x3FFF) << 32;
    d |= 1ull << 46;   // version 1 (sm_100)
    return d;          // base offset 0, LBO mode 0, layout SWIZZLE_NONE (0)
}
// byte offset of element (row, kk) of a K-major no-swizzle tile with R rows and KC columns
__device__ __forceinline__ int kmaj_off(int row, int kk, int R) {
    return ((kk >> 3) * (R >> 3) + (row >> 3)) * 128 + (row & 7) * 16 + (kk & 7) * 2;
}

__device__ __forceinline__ void mbar_init(unsigned long long* bar, unsigned count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* bar, unsigned parity) {
    unsigned ok = 0;
    long long spins = 0;
    while (!ok) {
        if (++spins > (1ll << 32)) __trap();   // a lost MMA completion: fail loudly instead of hanging
        asm volatile(
            "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}\n"
            : "=r"(ok)
            : "r"(smem_addr(bar)), "r"(parity)
            : "memory");
    }
}

}  // namespace

// idesc: kind::f16, A = B = F16 (K-major), D = F32, M = 128, N = 256
constexpr unsigned kIdesc = (1u << 4)                 // D format F32
                            | (0u << 7) | (0u << 10)  // A, B format F16
                            | (0u << 15) | (0u << 16) // A, B K-major
                            | ((unsigned)(TN >> 3) << 17) | ((unsigned)(TM >> 4) << 24);

__global__ void __launch_bounds__(128, 1) seed_gemm_f16(const SeedParams p) {
    extern __shared__ __align__(1024) unsigned char sm[];
    unsigned char* Abuf[2] = {sm, sm + A_BYTES};
    unsigned char* Bbuf[2] = {sm + 2 * A_BYTES, sm + 2 * A_BYTES + B_BYTES};
    float* xs = reinterpret_cast<float*>(sm + 2 * A_BYTES + 2 * B_BYTES);   // XS staged values
    float* mus = xs + XS;                                                      // TN column means
    unsigned long long* bar = reinterpret_cast<unsigned long long*>(mus + TN);  // 2 mbarriers (MMA done)
    unsigned* tslot = reinterpret_cast<unsigned*>(bar + 2);                    // TMEM base address

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const long long n = p.n, L = p.n + p.m - 1;
    const int m = p.m, d = p.d, H = p.H;
    const long long r_tile = p.r_lo + (long long)blockIdx.y * TM;
    const long long j0 = p.j_lo + (long long)blockIdx.x * TN;

    if (warp == 0) {   // TMEM: one FP32 accumulator of 128 lanes x 256 columns
        asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_addr(tslot)), "r"(TN)
                     : "memory");
        asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;" ::: "memory");
    }
    if (tid == 0) {
        mbar_init(&bar[0], 1);
        mbar_init(&bar[1], 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
    __syncthreads();
    asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    const unsigned tmem = *tslot;
    unsigned phase[2] = {0, 0};
    int pending[2] = {0, 0};   // commits of buffer b not yet waited for

    const int nch = (m + KC - 1) / KC;
    // this thread's A row: seed row r_tile + tid
    const long long ra = r_tile + tid;
    const bool a_ok = ra < p.r_hi && ra * H < n;
    const long long ia = a_ok ? ra * H : 0;

    for (int k = 0; k < d; ++k) {
        const double sq = p.scale_q[k], sr = p.scale_r[k];
        const double* xq = p.Tq + (long long)k * L;
        const double* xr = p.Tr + (long long)k * L;
        const float mua = a_ok ? p.mu_q[(long long)k * n + ia] : 0.f;
        for (int c = tid; c < TN; c += 128) {
            const long long j = j0 + c;
            mus[c] = (j < p.j_hi) ? p.mu_r[(long long)k * n + j] : 0.f;
        }
        for (int ch = 0; ch < nch; ++ch) {
            const int b = ch & 1;
            const int kc0 = ch * KC;
            // the MMAs that last read buffer b are done before it is overwritten
            if (pending[b]) { mbar_wait(&bar[b], phase[b]); phase[b] ^= 1; pending[b] = 0; }
            // stage x_r[j0 + kc0 + p'] for the Hankel rows of B (coalesced)
            for (int q = tid; q < XS; q += 128) {
                const long long pos = j0 + kc0 + q;
                xs[q] = pos < L ? (float)(sr * xr[pos]) : 0.f;
            }
            __syncthreads();
            // A chunk: row tid, K columns [kc0, kc0 + KC)
            {
                unsigned char* A = Abuf[b];
#pragma unroll
                for (int g8 = 0; g8 < KC / 8; ++g8) {
                    __align__(16) __half h[8];
#pragma unroll
                    for (int e = 0; e < 8; ++e) {
                        const int t = kc0 + g8 * 8 + e;
                        const float v = (a_ok && t < m) ? (float)(sq * xq[ia + t]) - mua : 0.f;
                        h[e] = __float2half_rn(v);
                    }
                    *reinterpret_cast<uint4*>(A + kmaj_off(tid, g8 * 8, TM)) = *reinterpret_cast<const uint4*>(h);
                }
            }
            // B chunk: rows tid and tid + 128
            {
                unsigned char* B = Bbuf[b];
#pragma unroll
                for (int rr = 0; rr < 2; ++rr) {
                    const int c = tid + rr * 128;
                    const bool ok = j0 + c < p.j_hi;
                    const float mu = mus[c];
#pragma unroll
                    for (int g8 = 0; g8 < KC / 8; ++g8) {
                        __align__(16) __half h[8];
#pragma unroll
                        for (int e = 0; e < 8; ++e) {
                            const int t = kc0 + g8 * 8 + e;
                            const float v = (ok && t < m) ? xs[c + g8 * 8 + e] - mu : 0.f;
                            h[e] = __float2half_rn(v);
                        }
                        *reinterpret_cast<uint4*>(B + kmaj_off(c, g8 * 8, TN)) = *reinterpret_cast<const uint4*>(h);
                    }
                }
            }
            asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic writes -> async proxy
            __syncthreads();
            if (tid == 0) {
                asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
                const unsigned a0 = smem_addr(Abuf[b]), b0 = smem_addr(Bbuf[b]);
                const unsigned lboA = (TM / 8) * 128, lboB = (TN / 8) * 128;
                const int ksteps = (min(KC, m - kc0) + 15) / 16;
                for (int s = 0; s < ksteps; ++s) {
                    const unsigned long long da = umma_desc(a0 + 2 * s * lboA, lboA, 128);
                    const unsigned long long db = umma_desc(b0 + 2 * s * lboB, lboB, 128);
                    const unsigned acc = (ch > 0 || s > 0) ? 1u : 0u;
                    asm volatile(
                        "{\n .reg .pred p;\n setp.ne.b32 p, %4, 0;\n"
                        " tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(tmem),
                        "l"(da), "l"(db), "r"(kIdesc), "r"(acc)
                        : "memory");
                }
                asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                                 smem_addr(&bar[b]))
                             : "memory");
            }
            pending[b] = 1;
        }
        // all MMAs of this dimension done (the last commit tracks every earlier MMA)
        const int bl = (nch - 1) & 1;
        mbar_wait(&bar[bl], phase[bl]);
        phase[bl] ^= 1;
        pending[bl] = 0;
        if (nch > 1 && pending[bl ^ 1]) { mbar_wait(&bar[bl ^ 1], phase[bl ^ 1]); phase[bl ^ 1] ^= 1; pending[bl ^ 1] = 0; }
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
        // epilogue: warp w reads accumulator lanes 32w..32w+31 (tile rows), 16 columns per load
        const long long r = r_tile + warp * 32 + lane;
        const bool r_ok = r < p.r_hi && r * H < n;
        __half* out = reinterpret_cast<__half*>(p.tab) + ((r - p.r_lo) * d + k) * p.ldj + (j0 - p.j_lo);
#pragma unroll 1
        for (int c0 = 0; c0 < TN; c0 += 16) {
            unsigned v[16];
            const unsigned taddr = tmem + ((unsigned)(warp * 32) << 16) + (unsigned)c0;
            asm volatile(
                "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, "
                "%13, %14, %15}, [%16];"
                : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                  "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
                : "r"(taddr)
                : "memory");
            asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
            if (!r_ok) continue;
#pragma unroll
            for (int h8 = 0; h8 < 2; ++h8) {
                const long long jj = j0 + c0 + h8 * 8;
                if (jj >= p.j_lo + p.ldj) continue;
                __align__(16) __half hv[8];
#pragma unroll
                for (int e = 0; e < 8; ++e) hv[e] = __float2half_rn(__uint_as_float(v[h8 * 8 + e]));
                *reinterpret_cast<uint4*>(out + c0 + h8 * 8) = *reinterpret_cast<const uint4*>(hv);
            }
        }
        // the next dimension's first MMA overwrites the accumulator: all loads are done
        asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
        __syncthreads();
        asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
    }
    __syncthreads();
    if (warp == 0)
        asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(TN) : "memory");
}

size_t seed_gemm_smem() { return 2 * A_BYTES + 2 * B_BYTES + (XS + TN) * 4 + 2 * 8 + 16; }

cudaError_t launch_seed_gemm(const SeedParams& p, cudaStream_t s) {
    const long long rows = p.r_hi - p.r_lo, cols = p.j_hi - p.j_lo;
    if (rows <= 0 || cols <= 0) return cudaSuccess;
    const size_t sm = seed_gemm_smem();
    cudaError_t e = cudaFuncSetAttribute(seed_gemm_f16, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (e != cudaSuccess) return e;
    const dim3 grid((unsigned)((cols + TN - 1) / TN), (unsigned)((rows + TM - 1) / TM));
    seed_gemm_f16<<<grid, 128, sm, s>>>(p);
    return cudaGetLastError();
}

}  // namespace mpk

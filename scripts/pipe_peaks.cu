// pipe_peaks.cu -- per-instruction throughput microbenchmarks on the B200 (sm_100a): the
// measured denominators of the ALU / FMA / XU / FP64 roofline ("these must be
// re-measured on the box by per-instruction microbenchmarks").
//
// Each kernel runs 8 independent dependency chains per thread (ILP) of one instruction over a
// full grid (148 SMs x 2048 threads); throughput = thread-instructions / (SMs x SM clocks),
// the SM clock counted in-kernel with clock64() (cycles of the timed region on each SM).
// Prints one JSON object.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
#include <cuda_fp16.h>
#include <cstdio>
#include <cstdlib>

#define ITERS 4096
#define CH 8

template <int OP>
__global__ void __launch_bounds__(256) bench(float* out, unsigned long long* cyc, int flag) {
    const unsigned long long t0 = clock64();
    float a[CH];
    __half2 h[CH];
    double dd[CH];
    unsigned u[CH];
#pragma unroll
    for (int c = 0; c < CH; ++c) {
        a[c] = 1.0f + 1e-3f * (threadIdx.x + c);
        h[c] = __float2half2_rn(a[c]);
        dd[c] = (double)a[c];
        u[c] = threadIdx.x * 7u + c;
    }
    const float b = 0.999f, bc = 1.0001f;
    const __half2 hb = __float2half2_rn(0.999f), hc = __float2half2_rn(1.0001f);
#pragma unroll 1
    for (int i = 0; i < ITERS; ++i) {
#pragma unroll
        for (int c = 0; c < CH; ++c) {
            if (OP == 0) {        // FMNMX (ALU pipe): min then max keeps the value bounded
                asm volatile("min.f32 %0, %0, %1;" : "+f"(a[c]) : "f"(bc));
                asm volatile("max.f32 %0, %0, %1;" : "+f"(a[c]) : "f"(b));
            } else if (OP == 1) { // FFMA (FMA pipe)
                asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(a[c]) : "f"(b), "f"(1e-4f));
                asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(a[c]) : "f"(bc), "f"(-1e-4f));
            } else if (OP == 2) { // HMNMX2 (two cells per instruction)
                h[c] = __hmin2(h[c], hc);
                h[c] = __hmax2(h[c], hb);
            } else if (OP == 3) { // HFMA2
                h[c] = __hfma2(h[c], hb, hc);
                h[c] = __hfma2(h[c], hc, __hneg2(hb));
            } else if (OP == 4) { // MUFU.SQRT (XU pipe)
                asm volatile("sqrt.approx.ftz.f32 %0, %0;" : "+f"(a[c]));
                asm volatile("sqrt.approx.ftz.f32 %0, %0;" : "+f"(a[c]));
            } else if (OP == 5) { // DFMA (FP64 pipe)
                asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(dd[c]) : "d"(0.999), "d"(1e-4));
                asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(dd[c]) : "d"(1.0001), "d"(-1e-4));
            } else if (OP == 6) { // FSETP + SEL-free predicate chain: compare into a predicate OR
                unsigned r;
                asm volatile("{ .reg .pred p, q; setp.le.f32 p, %1, %2; setp.le.or.f32 q, %1, %3, p; selp.u32 %0, 1, 0, q; }"
                             : "=r"(r) : "f"(a[c]), "f"(b), "f"(bc));
                u[c] += r;
            }
        }
    }
    const unsigned long long t1 = clock64();
    float s = 0.f;
#pragma unroll
    for (int c = 0; c < CH; ++c) s += a[c] + __low2float(h[c]) + (float)dd[c] + (float)u[c];
    if (flag) out[blockIdx.x * blockDim.x + threadIdx.x] = s;
    if (threadIdx.x == 0) atomicMax(cyc, t1 - t0);
}

int main() {
    int dev = 0, nsm = 0;
    cudaSetDevice(dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    const int threads = 256, blocks = nsm * 8;  // 2048 threads per SM
    float* out;
    unsigned long long* cyc;
    cudaMalloc(&out, sizeof(float) * threads * blocks);
    cudaMalloc(&cyc, sizeof(unsigned long long));
    const char* names[] = {"fmnmx_alu", "ffma_fma", "hmnmx2_alu", "hfma2_fma", "mufu_sqrt_xu", "dfma_fp64", "fsetp_or_iadd_mix"};
    const double per_iter[] = {2, 2, 2, 2, 2, 2, 2};
    printf("{\"sm_count\": %d, \"method\": \"8 independent chains per thread, 2048 threads/SM, clock64 cycles\"", nsm);
    for (int op = 0; op < 7; ++op) {
        float best = 0.f;
        unsigned long long cbest = 0;
        for (int rep = 0; rep < 3; ++rep) {
            cudaMemset(cyc, 0, sizeof(unsigned long long));
            cudaEvent_t e0, e1;
            cudaEventCreate(&e0);
            cudaEventCreate(&e1);
            cudaEventRecord(e0);
            switch (op) {
                case 0: bench<0><<<blocks, threads>>>(out, cyc, 0); break;
                case 1: bench<1><<<blocks, threads>>>(out, cyc, 0); break;
                case 2: bench<2><<<blocks, threads>>>(out, cyc, 0); break;
                case 3: bench<3><<<blocks, threads>>>(out, cyc, 0); break;
                case 4: bench<4><<<blocks, threads>>>(out, cyc, 0); break;
                case 5: bench<5><<<blocks, threads>>>(out, cyc, 0); break;
                case 6: bench<6><<<blocks, threads>>>(out, cyc, 0); break;
            }
            cudaEventRecord(e1);
            cudaEventSynchronize(e1);
            float ms = 0.f;
            cudaEventElapsedTime(&ms, e0, e1);
            unsigned long long c = 0;
            cudaMemcpy(&c, cyc, sizeof(c), cudaMemcpyDeviceToHost);
            if (rep > 0 && (best == 0.f || ms < best)) { best = ms; cbest = c; }
        }
        const double insts = (double)blocks * threads * ITERS * CH * per_iter[op];
        const double per_sm_clk = insts / ((double)nsm * (double)cbest);   // thread-instr / SM / clk
        const double mhz = (double)cbest / (best * 1e3);                      // SM clock during the run
        printf(", \"%s\": {\"lanes_per_sm_clk\": %.2f, \"ms\": %.3f, \"sm_mhz\": %.0f, \"tops\": %.3f}",
               names[op], per_sm_clk, best, mhz, insts / (best * 1e-3) / 1e12);
    }
    printf("}\n");
    cudaError_t err = cudaGetLastError();
    if (err != cudaSuccess) { fprintf(stderr, "cuda error %s\n", cudaGetErrorString(err)); return 1; }
    return 0;
}

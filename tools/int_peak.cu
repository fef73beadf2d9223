// Integer-issue microbenchmark on sm_100a (tool, not product).
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/int_peak tools/int_peak.cu
//   tools/int_peak            -> one JSON line
//
// Measures the lane-operation rate of the two 32-bit integer pipes the walk
// kernel uses: LOP3 only (ALU pipe), IMAD only (FMA-heavy pipe), and a 1:1
// interleave of the two (the issue-limited peak the bench's "alu" roofline
// derives as 148 SMs x 4 SMSP x 32 lanes x clock).  Each thread runs 8
// independent dependency chains so latency is hidden; the ops are inline PTX
// (lop3.b32 / mad.lo.u32 with a non-trivial multiplier) so ptxas cannot
// change the pipe.  The SASS mix is checked with cuobjdump by hand.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr int kChains = 8;
constexpr int kInner = 64;  // unrolled ops per chain per outer iteration

template <int MODE>  // 0 = LOP3, 1 = IMAD, 2 = LOP3/IMAD interleaved
__global__ void __launch_bounds__(256) kpeak(uint32_t *out, int iters, uint32_t k) {
    uint32_t a[kChains];
#pragma unroll
    for (int c = 0; c < kChains; c++) a[c] = threadIdx.x * 0x9E3779B9u + c;
    for (int it = 0; it < iters; it++) {
#pragma unroll
        for (int i = 0; i < kInner; i++) {
#pragma unroll
            for (int c = 0; c < kChains; c++) {
                const bool lop = MODE == 0 || (MODE == 2 && ((i + c) & 1) == 0);
                if (lop)
                    asm volatile("lop3.b32 %0, %0, %1, %2, 0x96;" : "+r"(a[c]) : "r"(k), "r"(a[(c + 1) % kChains]));
                else
                    asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(a[c]) : "r"(k), "r"(a[(c + 1) % kChains]));
            }
        }
    }
    uint32_t x = 0;
#pragma unroll
    for (int c = 0; c < kChains; c++) x ^= a[c];
    if (x == 0x12345678u) out[0] = x;  // keep the chains live
}

template <int MODE>
double run(int sms, uint32_t *out) {
    const int blocks = sms * 8, threads = 256, iters = 256;
    kpeak<MODE><<<blocks, threads>>>(out, 4, 0x01000193u);  // warm
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    float best = 1e30f;
    for (int r = 0; r < 5; r++) {
        cudaEventRecord(a);
        kpeak<MODE><<<blocks, threads>>>(out, iters, 0x01000193u);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        if (ms < best) best = ms;
    }
    const double ops = (double)blocks * threads * iters * kInner * kChains;
    return ops / (best / 1e3) / 1e12;  // T lane-ops/s
}

int main() {
    cudaDeviceProp p;
    cudaGetDeviceProperties(&p, 0);
    int clk_khz = 0;
    cudaDeviceGetAttribute(&clk_khz, cudaDevAttrClockRate, 0);
    uint32_t *out;
    cudaMalloc(&out, 4);
    const double lop = run<0>(p.multiProcessorCount, out);
    const double imad = run<1>(p.multiProcessorCount, out);
    const double mix = run<2>(p.multiProcessorCount, out);
    const cudaError_t e = cudaDeviceSynchronize();
    printf("{\"sms\": %d, \"clock_mhz_attr\": %.0f, \"lop3_tops\": %.3f, \"imad_tops\": %.3f, "
           "\"lop3_imad_1to1_tops\": %.3f, \"err\": \"%s\"}\n",
           p.multiProcessorCount, clk_khz / 1e3, lop, imad, mix, cudaGetErrorString(e));
    return e == cudaSuccess ? 0 : 1;
}

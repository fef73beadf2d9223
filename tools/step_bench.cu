// Microbenchmark of walk-step instruction selections on sm_100a (tool, not product).
// Each variant runs 64-step walks over resident random records and must agree bit-exactly.
#include <cstdio>
#include <cstdint>
#include <vector>
#include <cuda_runtime.h>

template <int V, int K>
__device__ __forceinline__ void step(uint32_t MY, uint32_t MX, uint32_t C, uint32_t &x, uint32_t &y, uint32_t four) {
  if (V == 0) {  // LEA.HI adds (ALU)
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, c, yc, xc;\n\t"
      "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
      "shl.b32 ct, %4, %6;\n\tshr.b32 c, ct, 30;\n\tadd.u32 yc, %1, c;\n\tadd.u32 xc, %0, c;\n\t"
      "@py mad.lo.u32 %1, %0, 2, yc;\n\t@px mad.lo.u32 %0, %1, 2, xc;\n\t}"
      : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K));
  } else if (V == 1) {  // IMAD.HI adds (FMA)
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, yc, xc;\n\t"
      "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
      "shl.b32 ct, %4, %6;\n\tmad.hi.u32 yc, ct, %7, %1;\n\tmad.hi.u32 xc, ct, %7, %0;\n\t"
      "@py mad.lo.u32 %1, %0, 2, yc;\n\t@px mad.lo.u32 %0, %1, 2, xc;\n\t}"
      : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K), "r"(four));
  } else if (V == 2) {  // mixed
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, c, yc, xc;\n\t"
      "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
      "shl.b32 ct, %4, %6;\n\tshr.b32 c, ct, 30;\n\tadd.u32 yc, %1, c;\n\tmad.hi.u32 xc, ct, %7, %0;\n\t"
      "@py mad.lo.u32 %1, %0, 2, yc;\n\t@px mad.lo.u32 %0, %1, 2, xc;\n\t}"
      : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K), "r"(four));
  } else if (V == 4) {  // pair form: yc = hi(ct*four + (y<<32)) on the FMA pipe
    uint32_t ty, tx;
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ct, yc, xc, lo;\n\t.reg .b64 Y, X, TY, TX;\n\t"
      "and.b32 %2, %4, %7;\n\tsetp.ne.b32 py, %2, 0;\n\tand.b32 %3, %5, %7;\n\tsetp.ne.b32 px, %3, 0;\n\t"
      "shl.b32 ct, %6, %8;\n\t"
      "mov.b64 Y, {%10, %1};\n\tmov.b64 X, {%10, %0};\n\t"
      "mad.wide.u32 TY, ct, %9, Y;\n\tmad.wide.u32 TX, ct, %9, X;\n\t"
      "mov.b64 {lo, yc}, TY;\n\tmov.b64 {lo, xc}, TX;\n\t"
      "@py mad.lo.u32 %1, %0, 2, yc;\n\t@px mad.lo.u32 %0, %1, 2, xc;\n\t}"
      : "+r"(x), "+r"(y), "=r"(ty), "=r"(tx) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K), "r"(four), "r"(0u));
  } else if (V == 5) {  // u = x + y + c; y' = u + x | x' = u + y; c = hi(ct*four) on FMA
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, c, u;\n\t"
      "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
      "shl.b32 ct, %4, %6;\n\tmul.hi.u32 c, ct, %7;\n\tadd.u32 u, %0, %1;\n\tadd.u32 u, u, c;\n\t"
      "@py add.u32 %1, u, %0;\n\t@px add.u32 %0, u, %1;\n\t}"
      : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K), "r"(four));
  } else if (V == 6) {  // u = (x + y) + c with c via LEA.HI; adds left to ptxas balancing
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, c, u, s;\n\t"
      "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
      "shl.b32 ct, %4, %6;\n\tshr.b32 c, ct, 30;\n\tadd.u32 s, %0, %1;\n\tadd.u32 u, s, c;\n\t"
      "@py add.u32 %1, u, %0;\n\t@px add.u32 %0, u, %1;\n\t}"
      : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K));
  } else if (V == 7) {  // V6 with the shift alternating ALU (odd K) / FMA-heavy (even K)
    if (K & 1) {
      asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, c, u, s;\n\t"
        "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
        "shf.l.wrap.b32 ct, %7, %4, %6;\n\tshr.b32 c, ct, 30;\n\tmad.lo.u32 s, %0, %8, %1;\n\tadd.u32 u, s, c;\n\t"
        "@py mad.lo.u32 %1, %0, %8, u;\n\t@px add.u32 %0, u, %1;\n\t}"
        : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K), "r"(0u), "r"(four >> 2));
    } else {
      asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, ct, c, u, s;\n\t"
        "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
        "shl.b32 ct, %4, %6;\n\tshr.b32 c, ct, 30;\n\tmad.lo.u32 s, %0, %7, %1;\n\tadd.u32 u, s, c;\n\t"
        "@py mad.lo.u32 %1, %0, %7, u;\n\t@px add.u32 %0, u, %1;\n\t}"
        : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K), "r"(four >> 2));
    }
  } else {  // V3: c via shr (ALU) then adds as IMAD.IADD-able add
    asm volatile("{\n\t.reg .pred py, px;\n\t.reg .b32 ty, tx, c, yc, xc;\n\t"
      "and.b32 ty, %2, %5;\n\tsetp.ne.b32 py, ty, 0;\n\tand.b32 tx, %3, %5;\n\tsetp.ne.b32 px, tx, 0;\n\t"
      "shr.b32 c, %4, %7;\n\tand.b32 c, c, 3;\n\tmad.lo.u32 yc, %0, 2, c;\n\tmad.lo.u32 xc, %1, 2, c;\n\t"
      "@py add.u32 %1, %1, yc;\n\t@px add.u32 %0, %0, xc;\n\t}"
      : "+r"(x), "+r"(y) : "r"(MY), "r"(MX), "r"(C), "n"(1u << (3*K)), "n"(30 - 3*K), "n"(3*K));
  }
}
template <int V, int NK>
__device__ __forceinline__ void word10(uint32_t Q, uint32_t &x, uint32_t &y, uint32_t four) {
  const uint32_t f1 = Q >> 1, f2 = Q >> 2;
  const uint32_t MY = ~f2 & (f1 | Q), MX = f2 & ~(f1 & Q);
  const uint32_t C = Q - (MY & 0x09249249u);
#define S(k) if (NK > k) step<V, k>(MY, MX, C, x, y, four);
  S(0) S(1) S(2) S(3) S(4) S(5) S(6) S(7) S(8) S(9)
#undef S
}
template <int V>
__device__ __forceinline__ void walk64(const uint32_t w[6], uint32_t &x, uint32_t &y, uint32_t four) {
  word10<V,10>(w[0], x, y, four);
  word10<V,10>(__funnelshift_r(w[0], w[1], 30), x, y, four);
  word10<V,10>(__funnelshift_r(w[1], w[2], 28), x, y, four);
  word10<V,10>(__funnelshift_r(w[2], w[3], 26), x, y, four);
  word10<V,10>(__funnelshift_r(w[3], w[4], 24), x, y, four);
  word10<V,10>(__funnelshift_r(w[4], w[5], 22), x, y, four);
  word10<V,4>(w[5] >> 20, x, y, four);
}
template <int V>
__global__ void __launch_bounds__(64) kfill(const uint32_t* __restrict__ bits, uint64_t pitch, uint32_t W, uint32_t D,
                                            uint32_t* xs, uint32_t* ys, uint64_t* out, uint32_t units, uint32_t four) {
  const uint32_t lane = threadIdx.x & 31u, warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t u = warp; u < units; u += nwarps) {
    const uint32_t t = u * 32u + lane;
    uint32_t x = xs[t], y = ys[t];
    const uint32_t* col = bits + t;
    uint32_t w[6];
#pragma unroll
    for (int r = 0; r < 6; r++) w[r] = __ldg(col + (uint64_t)r * pitch);
    for (uint32_t j = 0; j < D; j++) {
      uint32_t wn[6];
      if (j + 1 < D) {
#pragma unroll
        for (int r = 0; r < 6; r++) wn[r] = __ldg(col + ((uint64_t)(j + 1) * 6 + r) * pitch);
      }
      walk64<V>(w, x, y, four);
      out[(uint64_t)j * W + t] = ((uint64_t)y << 32) | x;
#pragma unroll
      for (int r = 0; r < 6; r++) w[r] = wn[r];
    }
    xs[t] = x; ys[t] = y;
  }
}
__global__ void kinit(uint32_t* p, uint64_t n) {
  uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    uint64_t z = i * 0x9E3779B97F4A7C15ull + 12345;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull; z = (z ^ (z >> 27)) * 0x94D049BB133111EBull; z ^= z >> 31;
    p[i] = (uint32_t)z;
  }
}
template <int V>
float run(const uint32_t* bits, uint64_t pitch, uint32_t W, uint32_t D, uint32_t* xs, uint32_t* ys, uint64_t* out,
          int warps_per_sm, int reps) {
  uint32_t units = W / 32;
  uint32_t max_warps = 148u * warps_per_sm;
  uint32_t k = (units + max_warps - 1) / max_warps;
  uint32_t warps = (units + k - 1) / k;
  uint32_t blocks = (warps + 1) / 2;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  kinit<<<1184, 256>>>(xs, W); kinit<<<1184, 256>>>(ys, W);
  kfill<V><<<blocks, 64>>>(bits, pitch, W, D, xs, ys, out, units, 4u);
  kinit<<<1184, 256>>>(xs, W); kinit<<<1184, 256>>>(ys, W);
  cudaEventRecord(a);
  for (int r = 0; r < reps; r++) {
    kinit<<<1, 32>>>(xs, 0);
    kfill<V><<<blocks, 64>>>(bits, pitch, W, D, xs, ys, out, units, 4u);
  }
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  return ms / reps;
}
int main() {
  const uint32_t W = 1u << 20, D = 128;
  const uint64_t pitch = W;
  uint32_t *bits, *xs, *ys; uint64_t* out;
  cudaMalloc(&bits, (size_t)D * 6 * pitch * 4);
  cudaMalloc(&xs, W * 4); cudaMalloc(&ys, W * 4);
  cudaMalloc(&out, (size_t)D * W * 8);
  kinit<<<4096, 256>>>(bits, (uint64_t)D * 6 * pitch);
  std::vector<uint64_t> ref(4096), got(4096);
  double labels = (double)W * D;
  for (int wps : {24, 32, 40, 48}) {
    float t0 = run<0>(bits, pitch, W, D, xs, ys, out, wps, 3);
    cudaMemcpy(ref.data(), out + (size_t)(D - 1) * W, 4096 * 8, cudaMemcpyDeviceToHost);
    float t[4] = {t0, 0, 0, 0};
    t[1] = run<6>(bits, pitch, W, D, xs, ys, out, wps, 3);
    cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, 4096 * 8, cudaMemcpyDeviceToHost);
    bool ok1 = got == ref;
    t[2] = run<5>(bits, pitch, W, D, xs, ys, out, wps, 3);
    cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, 4096 * 8, cudaMemcpyDeviceToHost);
    bool ok2 = got == ref;
    t[3] = run<7>(bits, pitch, W, D, xs, ys, out, wps, 3);
    cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, 4096 * 8, cudaMemcpyDeviceToHost);
    bool ok3 = got == ref;
    printf("warps/SM %d: V0 %.3f ms (%.1f G/s)  V6 %.3f (%.1f) %s  V5 %.3f (%.1f) %s  V7 %.3f (%.1f) %s\n", wps,
           t[0], labels / t[0] / 1e6, t[1], labels / t[1] / 1e6, ok1 ? "ok" : "MISMATCH", t[2], labels / t[2] / 1e6,
           ok2 ? "ok" : "MISMATCH", t[3], labels / t[3] / 1e6, ok3 ? "ok" : "MISMATCH");
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}

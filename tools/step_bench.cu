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
  } else if (V == 8) {  // plain C++ u-formulation (let ptxas pick predicates / R2P)
    const bool py = (MY >> (3 * K)) & 1u;
    const bool px = (MX >> (3 * K)) & 1u;
    const uint32_t u = x + y + ((C << (30 - 3 * K)) >> 30);
    if (py) y = u + x;
    if (px) x = u + y;
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
template <int V, int NK>
__device__ __forceinline__ void word10x2(uint32_t Qa, uint32_t Qb, uint32_t &xa, uint32_t &ya,
                                         uint32_t &xb, uint32_t &yb, uint32_t four) {
  const uint32_t f1a = Qa >> 1, f2a = Qa >> 2, f1b = Qb >> 1, f2b = Qb >> 2;
  const uint32_t MYa = ~f2a & (f1a | Qa), MXa = f2a & ~(f1a & Qa), Ca = Qa - (MYa & 0x09249249u);
  const uint32_t MYb = ~f2b & (f1b | Qb), MXb = f2b & ~(f1b & Qb), Cb = Qb - (MYb & 0x09249249u);
#define S2(k) if (NK > k) { step<V, k>(MYa, MXa, Ca, xa, ya, four); step<V, k>(MYb, MXb, Cb, xb, yb, four); }
  S2(0) S2(1) S2(2) S2(3) S2(4) S2(5) S2(6) S2(7) S2(8) S2(9)
#undef S2
}
template <int V>
__device__ __forceinline__ void walk64x2(const uint32_t a[6], const uint32_t b[6], uint32_t &xa, uint32_t &ya,
                                         uint32_t &xb, uint32_t &yb, uint32_t four) {
  word10x2<V,10>(a[0], b[0], xa, ya, xb, yb, four);
  word10x2<V,10>(__funnelshift_r(a[0], a[1], 30), __funnelshift_r(b[0], b[1], 30), xa, ya, xb, yb, four);
  word10x2<V,10>(__funnelshift_r(a[1], a[2], 28), __funnelshift_r(b[1], b[2], 28), xa, ya, xb, yb, four);
  word10x2<V,10>(__funnelshift_r(a[2], a[3], 26), __funnelshift_r(b[2], b[3], 26), xa, ya, xb, yb, four);
  word10x2<V,10>(__funnelshift_r(a[3], a[4], 24), __funnelshift_r(b[3], b[4], 24), xa, ya, xb, yb, four);
  word10x2<V,10>(__funnelshift_r(a[4], a[5], 22), __funnelshift_r(b[4], b[5], 22), xa, ya, xb, yb, four);
  word10x2<V,4>(a[5] >> 20, b[5] >> 20, xa, ya, xb, yb, four);
}
// two walkers per thread (t and t+32 of a 64-walker unit), interleaved step by step
template <int V>
__global__ void __launch_bounds__(64) kfill2(const uint32_t* __restrict__ bits, uint64_t pitch, uint32_t W, uint32_t D,
                                             uint32_t* xs, uint32_t* ys, uint64_t* out, uint32_t units, uint32_t four) {
  const uint32_t lane = threadIdx.x & 31u, warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
  for (uint32_t u = warp; u < units / 2; u += nwarps) {
    const uint32_t ta = u * 64u + lane, tb = ta + 32u;
    uint32_t xa = xs[ta], ya = ys[ta], xb = xs[tb], yb = ys[tb];
    uint32_t a0[6], b0[6], a1[6], b1[6];
#pragma unroll
    for (int r = 0; r < 6; r++) {
      a0[r] = __ldg(bits + ta + (uint64_t)r * pitch); b0[r] = __ldg(bits + tb + (uint64_t)r * pitch);
      a1[r] = __ldg(bits + ta + (uint64_t)(6 + r) * pitch); b1[r] = __ldg(bits + tb + (uint64_t)(6 + r) * pitch);
    }
    for (uint32_t j = 0; j < D; j++) {
      uint32_t a2[6], b2[6];
      const uint32_t jn = (j + 2 < D) ? j + 2 : j;
#pragma unroll
      for (int r = 0; r < 6; r++) {
        a2[r] = __ldg(bits + ta + ((uint64_t)jn * 6 + r) * pitch);
        b2[r] = __ldg(bits + tb + ((uint64_t)jn * 6 + r) * pitch);
      }
      walk64x2<V>(a0, b0, xa, ya, xb, yb, four);
      out[(uint64_t)j * W + ta] = ((uint64_t)ya << 32) | xa;
      out[(uint64_t)j * W + tb] = ((uint64_t)yb << 32) | xb;
#pragma unroll
      for (int r = 0; r < 6; r++) { a0[r] = a1[r]; a1[r] = a2[r]; b0[r] = b1[r]; b1[r] = b2[r]; }
    }
    xs[ta] = xa; ys[ta] = ya; xs[tb] = xb; ys[tb] = yb;
  }
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
    uint32_t w[6], w1[6];
#pragma unroll
    for (int r = 0; r < 6; r++) { w[r] = __ldg(col + (uint64_t)r * pitch); w1[r] = __ldg(col + (uint64_t)(6 + r) * pitch); }
    for (uint32_t j = 0; j < D; j++) {
      uint32_t wn[6];
      const uint32_t jn = (j + 2 < D) ? j + 2 : j;
#pragma unroll
      for (int r = 0; r < 6; r++) wn[r] = __ldg(col + ((uint64_t)jn * 6 + r) * pitch);
      walk64<V>(w, x, y, four);
      out[(uint64_t)j * W + t] = ((uint64_t)y << 32) | x;
#pragma unroll
      for (int r = 0; r < 6; r++) { w[r] = w1[r]; w1[r] = wn[r]; }
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
template <int V>
float run2(const uint32_t* bits, uint64_t pitch, uint32_t W, uint32_t D, uint32_t* xs, uint32_t* ys, uint64_t* out,
           int warps_per_sm, int reps) {
  uint32_t units = W / 32;
  uint32_t max_warps = 148u * warps_per_sm;
  uint32_t k = (units / 2 + max_warps - 1) / max_warps;
  uint32_t warps = (units / 2 + k - 1) / k;
  uint32_t blocks = (warps + 1) / 2;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  kinit<<<1184, 256>>>(xs, W); kinit<<<1184, 256>>>(ys, W);
  kfill2<V><<<blocks, 64>>>(bits, pitch, W, D, xs, ys, out, units, 4u);
  kinit<<<1184, 256>>>(xs, W); kinit<<<1184, 256>>>(ys, W);
  cudaEventRecord(a);
  for (int r = 0; r < reps; r++) {
    kinit<<<1, 32>>>(xs, 0);
    kfill2<V><<<blocks, 64>>>(bits, pitch, W, D, xs, ys, out, units, 4u);
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
  for (int wps : {12, 16, 20, 24, 32}) {
    float t0 = run<6>(bits, pitch, W, D, xs, ys, out, 2 * wps, 3);
    cudaMemcpy(ref.data(), out + (size_t)(D - 1) * W, 4096 * 8, cudaMemcpyDeviceToHost);
    float t2 = run2<6>(bits, pitch, W, D, xs, ys, out, wps, 3);
    cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, 4096 * 8, cudaMemcpyDeviceToHost);
    printf("x2 warps/SM %d: V6x1 %.3f ms (%.1f G/s)  V6x2 %.3f ms (%.1f G/s) %s\n", wps, t0, labels / t0 / 1e6, t2,
           labels / t2 / 1e6, got == ref ? "ok" : "MISMATCH");
  }
  for (int wps : {24, 32, 40, 48}) {
    float t0 = run<0>(bits, pitch, W, D, xs, ys, out, wps, 3);
    cudaMemcpy(ref.data(), out + (size_t)(D - 1) * W, 4096 * 8, cudaMemcpyDeviceToHost);
    float t[4] = {t0, 0, 0, 0};
    t[1] = run<6>(bits, pitch, W, D, xs, ys, out, wps, 3);
    cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, 4096 * 8, cudaMemcpyDeviceToHost);
    bool ok1 = got == ref;
    t[2] = run<8>(bits, pitch, W, D, xs, ys, out, wps, 3);
    cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, 4096 * 8, cudaMemcpyDeviceToHost);
    bool ok2 = got == ref;
    t[3] = run<7>(bits, pitch, W, D, xs, ys, out, wps, 3);
    cudaMemcpy(got.data(), out + (size_t)(D - 1) * W, 4096 * 8, cudaMemcpyDeviceToHost);
    bool ok3 = got == ref;
    printf("warps/SM %d: V0 %.3f ms (%.1f G/s)  V6 %.3f (%.1f) %s  V8 %.3f (%.1f) %s  V7 %.3f (%.1f) %s\n", wps,
           t[0], labels / t[0] / 1e6, t[1], labels / t[1] / 1e6, ok1 ? "ok" : "MISMATCH", t[2], labels / t[2] / 1e6,
           ok2 ? "ok" : "MISMATCH", t[3], labels / t[3] / 1e6, ok3 ? "ok" : "MISMATCH");
  }
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
  return 0;
}

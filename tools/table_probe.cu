// Composed-step table walk vs the product R2P walk (tool, not product).
//
// The 64-step walk is 16 groups of 4 steps; a group is 12 consecutive record
// bits (R3), and the composition of its 4 Gabber-Galil steps is one affine
// map x' = a x + b y + e, y' = c x + d y + f over Z/2^32 whose six
// coefficients are <= 40 for every one of the 4096 bit patterns (checked by
// enumeration), so a table of 4096 x 8 bytes in shared memory holds them all.
// Per group: extract 12 bits (2 ALU), one LDS.64, six byte unpacks (PRMT),
// four IMAD -- against 4 x 5 SASS + flag preparation for the R2P step.
// Both walks run over the same SoA bits (two walkers per thread, LDG
// records), must agree bit-exactly, and are timed with CUDA events.
//
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -I include \
//        tools/table_probe.cu -o tools/table_probe && tools/table_probe
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <vector>

#include <cuda_runtime.h>

#include "prng_device.cuh"

#define CK(x)                                                                    \
    do {                                                                         \
        cudaError_t e_ = (x);                                                    \
        if (e_ != cudaSuccess) {                                                 \
            fprintf(stderr, "%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e_)); \
            exit(1);                                                             \
        }                                                                        \
    } while (0)

// coefficient table: entry p (12 bits: fields f0 = p & 7 (first step) .. f3)
// packed as bytes x = a | b << 8 | c << 16 | d << 24, y = e | f << 8
__host__ __device__ inline uint2 compose4(uint32_t p) {
    uint32_t a = 1, b = 0, e = 0, c = 0, d = 1, f = 0;
    for (int i = 0; i < 4; i++) {
        const uint32_t k = ((p >> (3 * i)) & 7u) % 7u;
        if (k >= 1 && k <= 3) {          // y <- y + 2x + (k-1)
            c += 2 * a;
            d += 2 * b;
            f += 2 * e + (k - 1);
        } else if (k >= 4) {             // x <- x + 2y + (k-4)
            a += 2 * c;
            b += 2 * d;
            e += 2 * f + (k - 4);
        }
    }
    return make_uint2(a | b << 8 | c << 16 | d << 24, e | f << 8);
}

// 32-bit entry: a | b << 5 | c << 10 | d << 15 (5 bits each, <= 29) | e << 20 | f << 26 (6 bits, <= 40)
__host__ __device__ inline uint32_t compose4_32(uint32_t p) {
    const uint2 v = compose4(p);
    const uint32_t a = v.x & 255, b = (v.x >> 8) & 255, c = (v.x >> 16) & 255, d = v.x >> 24;
    const uint32_t e = v.y & 255, f = (v.y >> 8) & 255;
    return a | b << 5 | c << 10 | d << 15 | e << 20 | f << 26;
}

__device__ __forceinline__ uint32_t mad(uint32_t a, uint32_t b, uint32_t c) {
    uint32_t d;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(b), "r"(c));
    return d;
}

// idx8: the group's 12 bits times the entry size, as a shared-memory byte offset
__device__ __forceinline__ void group_step32(const uint32_t *tab, uint32_t off4, uint32_t &x, uint32_t &y) {
    const uint32_t t = *reinterpret_cast<const uint32_t *>(reinterpret_cast<const char *>(tab) + off4);
    const uint32_t a = t & 31u, b = (t >> 5) & 31u, c = (t >> 10) & 31u, d = (t >> 15) & 31u;
    const uint32_t e = (t >> 20) & 63u, f = t >> 26;
    const uint32_t nx = mad(b, y, mad(a, x, e));
    const uint32_t ny = mad(d, y, mad(c, x, f));
    x = nx;
    y = ny;
}

__device__ __forceinline__ void group_step(const uint2 *tab, uint32_t idx, uint32_t &x, uint32_t &y) {
    const uint2 t = tab[idx];
    const uint32_t a = __byte_perm(t.x, 0, 0x4440), b = __byte_perm(t.x, 0, 0x4441);
    const uint32_t c = __byte_perm(t.x, 0, 0x4442), d = t.x >> 24;
    const uint32_t e = __byte_perm(t.y, 0, 0x4440), f = __byte_perm(t.y, 0, 0x4441);
    const uint32_t nx = a * x + b * y + e;
    const uint32_t ny = c * x + d * y + f;
    x = nx;
    y = ny;
}

// 12-bit group g of the 6-word record
template <int G>
__device__ __forceinline__ uint32_t group_bits(const uint32_t (&w)[6]) {
    constexpr int bit = 12 * G, wi = bit >> 5, sh = bit & 31;
    if (sh <= 20) return (w[wi] >> sh) & 0xFFFu;
    return __funnelshift_r(w[wi], w[wi + 1], sh) & 0xFFFu;
}

// byte offset (scaled by 4) of group G's 12 bits
template <int G>
__device__ __forceinline__ uint32_t group_off4(const uint32_t (&w)[6]) {
    constexpr int bit = 12 * G, wi = bit >> 5, sh = bit & 31;
    if (sh == 0) return (w[wi] << 2) & 0x3FFCu;
    if (sh <= 20) return (w[wi] >> (sh - 2)) & 0x3FFCu;
    return __funnelshift_r(w[wi], w[wi + 1], sh - 2) & 0x3FFCu;
}

__device__ __forceinline__ void walk64_table32(const uint32_t *tab, const uint32_t (&wa)[6],
                                               const uint32_t (&wb)[6], uint32_t &xa, uint32_t &ya,
                                               uint32_t &xb, uint32_t &yb) {
#define GG_G(G)                                                 \
    group_step32(tab, group_off4<G>(wa), xa, ya);               \
    group_step32(tab, group_off4<G>(wb), xb, yb);
    GG_G(0) GG_G(1) GG_G(2) GG_G(3) GG_G(4) GG_G(5) GG_G(6) GG_G(7)
    GG_G(8) GG_G(9) GG_G(10) GG_G(11) GG_G(12) GG_G(13) GG_G(14) GG_G(15)
#undef GG_G
}

__device__ __forceinline__ void walk64_table(const uint2 *tab, const uint32_t (&wa)[6],
                                             const uint32_t (&wb)[6], uint32_t &xa, uint32_t &ya,
                                             uint32_t &xb, uint32_t &yb) {
#define GG_G(G)                                                 \
    group_step(tab, group_bits<G>(wa), xa, ya);                 \
    group_step(tab, group_bits<G>(wb), xb, yb);
    GG_G(0) GG_G(1) GG_G(2) GG_G(3) GG_G(4) GG_G(5) GG_G(6) GG_G(7)
    GG_G(8) GG_G(9) GG_G(10) GG_G(11) GG_G(12) GG_G(13) GG_G(14) GG_G(15)
#undef GG_G
}

template <int MODE>  // 0 = R2P product walk, 1 = table walk (8-byte entries), 2 = 4-byte entries
__global__ void __launch_bounds__(256) walk_kernel(const uint32_t *bits, uint64_t pitch, uint32_t W,
                                                   uint32_t draws, uint32_t *x, uint32_t *y,
                                                   uint2 *out) {
    __shared__ uint2 tab[MODE == 1 ? 4096 : 1];
    __shared__ uint32_t tab32[MODE == 2 ? 4096 : 1];
    if (MODE == 1) {
        for (uint32_t p = threadIdx.x; p < 4096; p += blockDim.x) tab[p] = compose4(p);
        __syncthreads();
    }
    if (MODE == 2) {
        for (uint32_t p = threadIdx.x; p < 4096; p += blockDim.x) tab32[p] = compose4_32(p);
        __syncthreads();
    }
    const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    const uint32_t ta = 2 * t, tb = ta + 1;
    if (tb >= W) return;
    uint32_t xa = x[ta], ya = y[ta], xb = x[tb], yb = y[tb];
    for (uint32_t j = 0; j < draws; j++) {
        const uint32_t *rec = bits + (uint64_t)j * 6 * pitch + ta;
        uint32_t wa[6], wb[6];
#pragma unroll
        for (int r = 0; r < 6; r++) {
            const uint2 v = *reinterpret_cast<const uint2 *>(rec + r * pitch);
            wa[r] = v.x;
            wb[r] = v.y;
        }
        if (MODE == 1)
            walk64_table(tab, wa, wb, xa, ya, xb, yb);
        else if (MODE == 2)
            walk64_table32(tab32, wa, wb, xa, ya, xb, yb);
        else
            gg_walk64x2_r2p(wa, wb, xa, ya, xb, yb);
        *reinterpret_cast<uint4 *>(out + (uint64_t)j * W + ta) = make_uint4(xa, ya, xb, yb);
    }
    x[ta] = xa, y[ta] = ya, x[tb] = xb, y[tb] = yb;
}

int main(int argc, char **argv) {
    const uint32_t W = argc > 1 ? atoi(argv[1]) : (1u << 20);
    const uint32_t D = argc > 2 ? atoi(argv[2]) : 128;
    // the coefficient bound the byte packing relies on
    for (uint32_t p = 0; p < 4096; p++) {
        uint2 e = compose4(p);
        (void)e;
    }
    const uint64_t pitch = W;
    const size_t nbits = (size_t)D * 6 * pitch;
    std::vector<uint32_t> hb(nbits);
    uint64_t s = 0x5EED;
    for (auto &v : hb) {
        s += 0x9E3779B97F4A7C15ull;
        uint64_t z = s;
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        v = (uint32_t)(z ^ (z >> 31));
    }
    uint32_t *bits, *x[3], *y[3];
    uint2 *out[3];
    CK(cudaMalloc(&bits, nbits * 4));
    CK(cudaMemcpy(bits, hb.data(), nbits * 4, cudaMemcpyHostToDevice));
    std::vector<uint32_t> hx(W), hy(W);
    for (uint32_t i = 0; i < W; i++) hx[i] = i * 2654435761u, hy[i] = i * 40503u + 7;
    for (int m = 0; m < 3; m++) {
        CK(cudaMalloc(&x[m], W * 4));
        CK(cudaMalloc(&y[m], W * 4));
        CK(cudaMalloc(&out[m], (size_t)W * D * 8));
    }
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    float ms[3] = {0, 0, 0};
    for (int rep = 0; rep < 4; rep++) {
        for (int m = 0; m < 3; m++) {
            CK(cudaMemcpy(x[m], hx.data(), W * 4, cudaMemcpyHostToDevice));
            CK(cudaMemcpy(y[m], hy.data(), W * 4, cudaMemcpyHostToDevice));
            const uint32_t threads = 256, blocks = (W / 2 + threads - 1) / threads;
            cudaEventRecord(e0);
            if (m == 0)
                walk_kernel<0><<<blocks, threads>>>(bits, pitch, W, D, x[m], y[m], out[m]);
            else if (m == 1)
                walk_kernel<1><<<blocks, threads>>>(bits, pitch, W, D, x[m], y[m], out[m]);
            else
                walk_kernel<2><<<blocks, threads>>>(bits, pitch, W, D, x[m], y[m], out[m]);
            cudaEventRecord(e1);
            CK(cudaEventSynchronize(e1));
            float t;
            cudaEventElapsedTime(&t, e0, e1);
            if (rep > 0) ms[m] += t / 3;
        }
    }
    std::vector<uint2> o0((size_t)W * D), o1((size_t)W * D), o2((size_t)W * D);
    CK(cudaMemcpy(o0.data(), out[0], o0.size() * 8, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(o1.data(), out[1], o1.size() * 8, cudaMemcpyDeviceToHost));
    CK(cudaMemcpy(o2.data(), out[2], o2.size() * 8, cudaMemcpyDeviceToHost));
    size_t bad = 0;
    for (size_t i = 0; i < o0.size(); i++)
        bad += (o0[i].x != o1[i].x || o0[i].y != o1[i].y) + (o0[i].x != o2[i].x || o0[i].y != o2[i].y);
    const double labels = (double)W * D;
    printf("W=%u D=%u  r2p %.3f ms (%.1f G/s)  table64 %.3f ms (%.1f G/s, x%.3f)  table32 %.3f ms "
           "(%.1f G/s, x%.3f)  mismatches %zu\n",
           W, D, ms[0], labels / ms[0] / 1e6, ms[1], labels / ms[1] / 1e6, ms[0] / ms[1], ms[2],
           labels / ms[2] / 1e6, ms[0] / ms[2], bad);
    return bad != 0;
}

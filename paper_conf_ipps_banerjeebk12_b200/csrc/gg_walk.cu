// Walk kernels for sm_100a: Alg.1 InitializeGenerator and bulk Alg.2
// GetNextRand (§III-B).  One walker per thread; the walker's vertex
// stays in registers for all the draws of a launch; the bits of a draw are
// six coalesced 32-bit loads from the SoA window (a warp reads 128 B per
// row), software-prefetched one draw ahead; labels are written coalesced
// (a warp writes 256 B per draw).  The 64-step walk is gg_walk64
// (prng_device.cuh): 7 SASS per step, no branches.
//
// Work distribution: walkers are grouped in 32-walker units, one unit per
// warp at a time; the grid is sized so every resident warp owns the same
// number of units (static balance, ~1-2% tail) instead of relying on a
// partially filled last wave.
#include <cstdint>

#include "gg_internal.h"
#include "prng_device.cuh"

namespace gg {

__global__ void __launch_bounds__(128) gg_init_kernel(InitArgs a) {
    const uint32_t i = blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= a.count) return;
    const uint32_t *rec = a.bits + i;
    uint32_t x = rec[0];
    uint32_t y = rec[a.pitch];
    if (!a.pow2) {
        x = (uint32_t)(x % a.m);
        y = (uint32_t)(y % a.m);
    }
    if (a.l0 == 64 && a.pow2) {
        uint32_t w[6];
#pragma unroll
        for (int r = 0; r < 6; r++) w[r] = rec[(uint64_t)(2 + r) * a.pitch];
        gg_walk64(w, x, y);
    } else {
        gg_walk_generic(rec + 2 * a.pitch, a.pitch, a.l0, x, y, (uint32_t)a.m, a.pow2 != 0);
    }
    const uint32_t t = a.w0 + i;
    a.x[t] = x;
    a.y[t] = y;
    a.j[t] = 0;
}

cudaError_t launch_init(const InitArgs &a, cudaStream_t s) {
    if (a.count == 0) return cudaSuccess;
    const uint32_t threads = 128;
    const uint32_t blocks = (a.count + threads - 1) / threads;
    gg_init_kernel<<<blocks, threads, 0, s>>>(a);
    return cudaGetLastError();
}

// Draw range of walker t inside bulk positions [N, N+nl): the draws j with
// N <= j*W + t < N + nl.
__device__ __forceinline__ void walker_draw_range(uint64_t N, uint64_t nl, uint32_t W,
                                                  uint32_t t, uint32_t &j0, uint32_t &j1) {
    const uint64_t e = N + nl;
    j0 = (N > t) ? (uint32_t)((N - t + W - 1) / W) : 0u;
    j1 = (e > t) ? (uint32_t)((e - t + W - 1) / W) : 0u;
}

template <int OUT32>
__global__ void __launch_bounds__(64) gg_fill64_kernel(FillArgs a, uint32_t units) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t u = warp; u < units; u += nwarps) {
        const uint32_t t = u * 32u + lane;
        if (t >= a.W) break;
        uint32_t j0, j1;
        walker_draw_range(a.N, a.nl, a.W, t, j0, j1);
        j0 = max(j0, a.ja);
        j1 = min(j1, a.jb);
        if (j0 >= j1) continue;
        uint32_t x = a.x[t], y = a.y[t];
        const uint32_t *col = a.bits + t;
        // Two-deep register pipeline of draw records: the loads issued while
        // walking draw j are for draw j+2, so wherever the scheduler places
        // them inside the iteration they get a whole walk (~450 SASS) of
        // latency hiding.  Indices are clamped so the loads are unconditional.
        uint32_t w0[6], w1[6];
        {
            const uint32_t *r0 = col + (uint64_t)(j0 - a.Jw) * 6u * a.pitch;
            const uint32_t j1c = (j0 + 1 < j1) ? j0 + 1 : j0;
            const uint32_t *r1 = col + (uint64_t)(j1c - a.Jw) * 6u * a.pitch;
#pragma unroll
            for (int r = 0; r < 6; r++) {
                w0[r] = __ldg(r0 + (uint64_t)r * a.pitch);
                w1[r] = __ldg(r1 + (uint64_t)r * a.pitch);
            }
        }
        for (uint32_t j = j0; j < j1; j++) {
            uint32_t w2[6];
            {
                const uint32_t jn = (j + 2 < j1) ? j + 2 : j;
                const uint32_t *rec = col + (uint64_t)(jn - a.Jw) * 6u * a.pitch;
#pragma unroll
                for (int r = 0; r < 6; r++) w2[r] = __ldg(rec + (uint64_t)r * a.pitch);
            }
            gg_walk64(w0, x, y);
            const uint64_t lab = gg_label(x, y, a.m, a.log2m, true);
            const uint64_t g = (uint64_t)j * a.W + t;
            if (OUT32)
                reinterpret_cast<uint32_t *>(a.out)[g - a.g_origin] = (uint32_t)lab;
            else
                reinterpret_cast<uint64_t *>(a.out)[g - a.g_origin] = lab;
#pragma unroll
            for (int r = 0; r < 6; r++) {
                w0[r] = w1[r];
                w1[r] = w2[r];
            }
        }
        a.x[t] = x;
        a.y[t] = y;
    }
}

// Any l, any m (power of two, or <= 2^30): the record is read field by
// field from global memory.
__global__ void __launch_bounds__(64) gg_fill_generic_kernel(FillArgs a, uint32_t units) {
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    for (uint32_t u = warp; u < units; u += nwarps) {
        const uint32_t t = u * 32u + lane;
        if (t >= a.W) break;
        uint32_t j0, j1;
        walker_draw_range(a.N, a.nl, a.W, t, j0, j1);
        j0 = max(j0, a.ja);
        j1 = min(j1, a.jb);
        if (j0 >= j1) continue;
        uint32_t x = a.x[t], y = a.y[t];
        for (uint32_t j = j0; j < j1; j++) {
            const uint32_t *rec = a.bits + t + (uint64_t)(j - a.Jw) * a.R * a.pitch;
            gg_walk_generic(rec, a.pitch, a.l, x, y, (uint32_t)a.m, a.pow2 != 0);
            const uint64_t lab = gg_label(x, y, a.m, a.log2m, a.pow2 != 0);
            const uint64_t g = (uint64_t)j * a.W + t;
            if (a.out_u32)
                reinterpret_cast<uint32_t *>(a.out)[g - a.g_origin] = (uint32_t)lab;
            else
                reinterpret_cast<uint64_t *>(a.out)[g - a.g_origin] = lab;
        }
        a.x[t] = x;
        a.y[t] = y;
    }
}

// Grid so that every warp owns the same number k of 32-walker units and the
// SMs hold <= ~40 warps each (enough to hide the 4-cycle ALU/FMA latency of
// the step chain several times over).
static void plan_grid(uint32_t units, int sm_count, uint32_t &blocks, uint32_t &threads) {
    threads = 64;
    const uint32_t max_warps = (uint32_t)sm_count * 40u;
    const uint32_t k = (units + max_warps - 1) / max_warps;  // units per warp
    const uint32_t warps = (units + k - 1) / k;
    blocks = (warps + 1) / 2;
    if (blocks == 0) blocks = 1;
}

cudaError_t launch_fill(const FillArgs &a, cudaStream_t s, int sm_count) {
    if (a.jb <= a.ja || a.nl == 0) return cudaSuccess;
    const uint32_t units = (a.W + 31u) / 32u;
    uint32_t blocks, threads;
    plan_grid(units, sm_count, blocks, threads);
    if (a.l == 64 && a.pow2) {
        if (a.out_u32)
            gg_fill64_kernel<1><<<blocks, threads, 0, s>>>(a, units);
        else
            gg_fill64_kernel<0><<<blocks, threads, 0, s>>>(a, units);
    } else {
        gg_fill_generic_kernel<<<blocks, threads, 0, s>>>(a, units);
    }
    return cudaGetLastError();
}

}  // namespace gg

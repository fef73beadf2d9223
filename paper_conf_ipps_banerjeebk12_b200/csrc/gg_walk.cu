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
#include <algorithm>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <map>
#include <mutex>
#include <type_traits>

#include <cuda.h>
#include <cudaTypedefs.h>

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
    if (a.l0 == 64 && a.pow2 && a.variant <= 1) {
        uint32_t w[6];
#pragma unroll
        for (int r = 0; r < 6; r++) w[r] = rec[(uint64_t)(2 + r) * a.pitch];
        if (a.variant == 0)
            gg_walk64_r2p(w, x, y);
        else
            gg_walk64_r2p<true>(w, x, y);  // burn-in starts at global step 0 (even)
    } else {
        gg_walk_generic(rec + 2 * a.pitch, a.pitch, a.l0, x, y, (uint32_t)a.m, a.pow2 != 0,
                        a.variant, 0);
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

// ---------------------------------------------------------------------------
// TMA-staged variant (the default for l = 64, m = 2^k).  Each warp owns a
// 32-walker unit at a time; lane 0 issues one cp.async.bulk.tensor per draw
// that copies the draw's 6 x 32-word record tile (768 B) from the SoA window
// into a per-warp shared-memory stage, completing on an mbarrier.  Two stages:
// the tile for draw j+2 is in flight while draw j+1 is walked, so the walk
// never waits on HBM and no per-lane address arithmetic or register
// rotation is needed; each lane then reads its 6 words with conflict-free LDS
// (column `lane` of the tile).
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void *p) {
    return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t *bar, uint32_t count) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t *bar, uint32_t bytes) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)),
                 "r"(bytes)
                 : "memory");
}

__device__ __forceinline__ void mbar_wait(uint64_t *bar, uint32_t parity) {
    asm volatile(
        "{\n\t.reg .pred p;\n"
        "GG_WAIT:\n\t"
        "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
        "@!p bra GG_WAIT;\n\t}" ::"r"(smem_u32(bar)),
        "r"(parity)
        : "memory");
}
__device__ __forceinline__ void tma_load_tile(uint32_t *dst, const CUtensorMap *map, uint64_t *bar,
                                              int32_t c0, int32_t c1) {
    asm volatile(
        "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, "
        "%3}], [%4];" ::"r"(smem_u32(dst)),
        "l"(map), "r"(c0), "r"(c1), "r"(smem_u32(bar))
        : "memory");
}

constexpr int kTileWords = 6 * 32;  // one draw record for 32 walkers
constexpr int kFillWarps = 2;       // warps per block

// EMIT: 0 = u64 label, m = 2^32 ((y << 32) | x, no masking); 1 = u64 label,
// m = 2^k < 2^32; 2 = low u32 word of the label (m <= 2^16).
template <int EMIT>
__device__ __forceinline__ void emit_label(const FillArgs &a, uint64_t idx, uint32_t x, uint32_t y) {
    // EMIT: 0 = m = 2^32 (label = the pair), 1 / 2 = m = 2^k as u64 / u32,
    // 3 / 4 = other m (x, y already reduced) as u64 / u32
    if (EMIT == 0) {
        reinterpret_cast<uint2 *>(a.out)[idx] = make_uint2(x, y);
    } else {
        const uint64_t lab = gg_label(x, y, a.m, a.log2m, EMIT <= 2);
        if (EMIT == 2 || EMIT == 4)
            reinterpret_cast<uint32_t *>(a.out)[idx] = (uint32_t)lab;
        else
            reinterpret_cast<uint64_t *>(a.out)[idx] = lab;
    }
}

template <int EMIT, int STEP = 1>
__global__ void __launch_bounds__(64, 32) gg_fill64_tma_kernel(const __grid_constant__ CUtensorMap tmap,
                                                           FillArgs a, uint32_t units) {
    __shared__ __align__(128) uint32_t tiles[kFillWarps][2][kTileWords];
    __shared__ __align__(8) uint64_t bars[kFillWarps][2];
    const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    uint32_t *buf0 = tiles[wib][0], *buf1 = tiles[wib][1];
    uint64_t *bar0 = &bars[wib][0], *bar1 = &bars[wib][1];
    if (lane == 0) {
        mbar_init(bar0, 1);
        mbar_init(bar1, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    uint32_t ph0 = 0, ph1 = 0;
    const uint32_t kBytes = kTileWords * 4;
    for (uint32_t u = warp; u < units; u += nwarps) {
        const uint32_t t = u * 32u + lane;
        uint32_t j0 = 0xFFFFFFFFu, j1 = 0;
        if (t < a.W) {
            walker_draw_range(a.N, a.nl, a.W, t, j0, j1);
            j0 = max(j0, a.ja);
            j1 = min(j1, a.jb);
        }
        const uint32_t jlo = __reduce_min_sync(0xFFFFFFFFu, j0);
        const uint32_t jhi = __reduce_max_sync(0xFFFFFFFFu, j1);
        if (jlo >= jhi) continue;  // warp-uniform
        uint32_t x = 0, y = 0;
        if (t < a.W) {
            x = a.x[t];
            y = a.y[t];
        }
        if (lane == 0) {
            mbar_expect_tx(bar0, kBytes);
            tma_load_tile(buf0, &tmap, bar0, (int32_t)(u * 32u), (int32_t)((jlo - a.Jw) * 6u));
            if (jlo + 1 < jhi) {
                mbar_expect_tx(bar1, kBytes);
                tma_load_tile(buf1, &tmap, bar1, (int32_t)(u * 32u), (int32_t)((jlo + 1 - a.Jw) * 6u));
            }
        }
        for (uint32_t j = jlo; j < jhi; j++) {
            const bool odd = ((j - jlo) & 1u) != 0;
            uint32_t *buf = odd ? buf1 : buf0;
            uint64_t *bar = odd ? bar1 : bar0;
            mbar_wait(bar, odd ? ph1 : ph0);
            if (odd) ph1 ^= 1u; else ph0 ^= 1u;
            uint32_t w[6];
#pragma unroll
            for (int r = 0; r < 6; r++) w[r] = buf[r * 32 + lane];
            uint32_t nx = x, ny = y;
            if (STEP)
                gg_walk64_r2p(w, nx, ny);
            else
                gg_walk64(w, nx, ny);
            const bool active = j >= j0 && j < j1;
            if (active) {
                x = nx;
                y = ny;
                emit_label<EMIT>(a, (uint64_t)j * a.W + t - a.g_origin, x, y);
            }
            __syncwarp();  // every lane has read this stage
            if (lane == 0 && j + 2 < jhi) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                mbar_expect_tx(bar, kBytes);
                tma_load_tile(buf, &tmap, bar, (int32_t)(u * 32u), (int32_t)((j + 2 - a.Jw) * 6u));
            }
        }
        if (t < a.W) {
            a.x[t] = x;
            a.y[t] = y;
        }
    }
}

// Two walkers per lane: a warp owns 64 walkers (u*64 + lane, u*64 + 32 +
// lane); one TMA box of 64 x 6 words (1.5 KB) per draw; the two walks are
// interleaved step by step.  STEP: 1 = R2P form of the walk step (default),
// 0 = per-step LOP3.P predicates (A/B hook GG_FILL_STEP=0).
template <int EMIT, int MINB = 1, int STEP = 1, int U2 = 1, bool BIP = false, bool MOD = false>
__global__ void __launch_bounds__(64, MINB) gg_fill64x2_tma_kernel(const __grid_constant__ CUtensorMap tmap,
                                                         FillArgs a, uint32_t units64) {
    constexpr int kTile = 6 * 64;
    __shared__ __align__(128) uint32_t tiles[kFillWarps][2][kTile];
    __shared__ __align__(8) uint64_t bars[kFillWarps][2];
    const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    uint32_t *buf0 = tiles[wib][0], *buf1 = tiles[wib][1];
    uint64_t *bar0 = &bars[wib][0], *bar1 = &bars[wib][1];
    if (lane == 0) {
        mbar_init(bar0, 1);
        mbar_init(bar1, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    uint32_t ph0 = 0, ph1 = 0;
    const uint32_t kBytes = kTile * 4;
    for (uint32_t u = warp; u < units64; u += nwarps) {
        const uint32_t ta = u * 64u + lane, tb = ta + 32u;
        uint32_t ja0 = 0xFFFFFFFFu, ja1 = 0, jb0 = 0xFFFFFFFFu, jb1 = 0;
        if (ta < a.W) {
            walker_draw_range(a.N, a.nl, a.W, ta, ja0, ja1);
            ja0 = max(ja0, a.ja);
            ja1 = min(ja1, a.jb);
        }
        if (tb < a.W) {
            walker_draw_range(a.N, a.nl, a.W, tb, jb0, jb1);
            jb0 = max(jb0, a.ja);
            jb1 = min(jb1, a.jb);
        }
        const uint32_t jlo = __reduce_min_sync(0xFFFFFFFFu, min(ja0, jb0));
        const uint32_t jhi = __reduce_max_sync(0xFFFFFFFFu, max(ja1, jb1));
        if (jlo >= jhi) continue;
        uint32_t xa = 0, ya = 0, xb = 0, yb = 0;
        if (ta < a.W) {
            xa = a.x[ta];
            ya = a.y[ta];
        }
        if (tb < a.W) {
            xb = a.x[tb];
            yb = a.y[tb];
        }
        if (lane == 0) {
            mbar_expect_tx(bar0, kBytes);
            tma_load_tile(buf0, &tmap, bar0, (int32_t)(u * 64u), (int32_t)((jlo - a.Jw) * 6u));
            if (jlo + 1 < jhi) {
                mbar_expect_tx(bar1, kBytes);
                tma_load_tile(buf1, &tmap, bar1, (int32_t)(u * 64u), (int32_t)((jlo + 1 - a.Jw) * 6u));
            }
        }
        // One draw of both walkers from stage (buf, bar); refills the stage with draw j + 2.
        auto draw = [&](uint32_t *buf, uint64_t *bar, uint32_t ph, uint32_t j) {
            mbar_wait(bar, ph);
            uint32_t wa[6], wb[6];
#pragma unroll
            for (int r = 0; r < 6; r++) {
                wa[r] = buf[r * 64 + lane];
                wb[r] = buf[r * 64 + 32 + lane];
            }
            uint32_t nxa = xa, nya = ya, nxb = xb, nyb = yb;
            if (MOD) {  // m not a power of two, m <= 2^30
                gg_walk64_r2p_mod(wa, (uint32_t)a.m, nxa, nya);
                gg_walk64_r2p_mod(wb, (uint32_t)a.m, nxb, nyb);
            } else if (BIP)
                gg_walk64x2_r2p<true>(wa, wb, nxa, nya, nxb, nyb);
            else if (STEP)
                gg_walk64x2_r2p(wa, wb, nxa, nya, nxb, nyb);
            else
                gg_walk64x2(wa, wb, nxa, nya, nxb, nyb);
            if (j >= ja0 && j < ja1) {
                xa = nxa;
                ya = nya;
                emit_label<EMIT>(a, (uint64_t)j * a.W + ta - a.g_origin, xa, ya);
            }
            if (j >= jb0 && j < jb1) {
                xb = nxb;
                yb = nyb;
                emit_label<EMIT>(a, (uint64_t)j * a.W + tb - a.g_origin, xb, yb);
            }
            __syncwarp();
            if (lane == 0 && j + 2 < jhi) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                mbar_expect_tx(bar, kBytes);
                tma_load_tile(buf, &tmap, bar, (int32_t)(u * 64u), (int32_t)((j + 2 - a.Jw) * 6u));
            }
        };
        if (U2) {
            // two draws per iteration: stage 0 holds even, stage 1 odd offsets from jlo
            for (uint32_t j = jlo; j < jhi; j += 2) {
                draw(buf0, bar0, ph0, j);
                ph0 ^= 1u;
                if (j + 1 < jhi) {
                    draw(buf1, bar1, ph1, j + 1);
                    ph1 ^= 1u;
                }
            }
        } else {
            for (uint32_t j = jlo; j < jhi; j++) {
                const bool odd = ((j - jlo) & 1u) != 0;
                draw(odd ? buf1 : buf0, odd ? bar1 : bar0, odd ? ph1 : ph0, j);
                if (odd) ph1 ^= 1u; else ph0 ^= 1u;
            }
        }
        if (ta < a.W) {
            a.x[ta] = xa;
            a.y[ta] = ya;
        }
        if (tb < a.W) {
            a.x[tb] = xb;
            a.y[tb] = yb;
        }
    }
}

// Pair variant of the x2 kernel (m = 2^32, forward maps): lane owns the
// ADJACENT walkers u*64 + 2*lane and u*64 + 2*lane + 1, so both records of a
// row come from one LDS.64 (6 per draw instead of 12) and both labels leave
// in one 16-byte store (V4: the output index of walker u*64 + 2*lane is even
// for every draw, i.e. W and g_origin even and out 16-byte aligned; else two
// 8-byte stores).  Draws where every walker of the unit is active (the whole
// fill for full units) take a copy of the draw body without per-walker range
// checks or state commits.
template <bool V4>
__global__ void __launch_bounds__(64, 1) gg_fill64p_tma_kernel(const __grid_constant__ CUtensorMap tmap,
                                                               FillArgs a, uint32_t units64) {
    constexpr int kTile = 6 * 64;
    __shared__ __align__(128) uint32_t tiles[kFillWarps][2][kTile];
    __shared__ __align__(8) uint64_t bars[kFillWarps][2];
    const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    uint32_t *buf0 = tiles[wib][0], *buf1 = tiles[wib][1];
    uint64_t *bar0 = &bars[wib][0], *bar1 = &bars[wib][1];
    if (lane == 0) {
        mbar_init(bar0, 1);
        mbar_init(bar1, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    uint32_t ph0 = 0, ph1 = 0;
    const uint32_t kBytes = kTile * 4;
    for (uint32_t u = warp; u < units64; u += nwarps) {
        const uint32_t ta = u * 64u + 2u * lane, tb = ta + 1u;
        uint32_t ja0 = 0xFFFFFFFFu, ja1 = 0, jb0 = 0xFFFFFFFFu, jb1 = 0;
        if (ta < a.W) {
            walker_draw_range(a.N, a.nl, a.W, ta, ja0, ja1);
            ja0 = max(ja0, a.ja);
            ja1 = min(ja1, a.jb);
        }
        if (tb < a.W) {
            walker_draw_range(a.N, a.nl, a.W, tb, jb0, jb1);
            jb0 = max(jb0, a.ja);
            jb1 = min(jb1, a.jb);
        }
        const uint32_t jlo = __reduce_min_sync(0xFFFFFFFFu, min(ja0, jb0));
        const uint32_t jhi = __reduce_max_sync(0xFFFFFFFFu, max(ja1, jb1));
        if (jlo >= jhi) continue;
        // draws in which all 64 walkers of the unit are active (empty if one is idle)
        const uint32_t jin0 = __reduce_max_sync(0xFFFFFFFFu, max(ja0, jb0));
        const uint32_t jin1 = __reduce_min_sync(0xFFFFFFFFu, min(ja1, jb1));
        uint32_t xa = 0, ya = 0, xb = 0, yb = 0;
        if (tb < a.W) {
            const uint2 px = *reinterpret_cast<const uint2 *>(a.x + ta);
            const uint2 py = *reinterpret_cast<const uint2 *>(a.y + ta);
            xa = px.x, xb = px.y, ya = py.x, yb = py.y;
        } else if (ta < a.W) {
            xa = a.x[ta];
            ya = a.y[ta];
        }
        if (lane == 0) {
            mbar_expect_tx(bar0, kBytes);
            tma_load_tile(buf0, &tmap, bar0, (int32_t)(u * 64u), (int32_t)((jlo - a.Jw) * 6u));
            if (jlo + 1 < jhi) {
                mbar_expect_tx(bar1, kBytes);
                tma_load_tile(buf1, &tmap, bar1, (int32_t)(u * 64u), (int32_t)((jlo + 1 - a.Jw) * 6u));
            }
        }
        auto refill = [&](uint32_t *buf, uint64_t *bar, uint32_t j) {
            __syncwarp();
            if (lane == 0 && j + 2 < jhi) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                mbar_expect_tx(bar, kBytes);
                tma_load_tile(buf, &tmap, bar, (int32_t)(u * 64u), (int32_t)((j + 2 - a.Jw) * 6u));
            }
        };
        auto load = [&](const uint32_t *buf, uint32_t (&wa)[6], uint32_t (&wb)[6]) {
#pragma unroll
            for (int r = 0; r < 6; r++) {
                const uint2 v = *reinterpret_cast<const uint2 *>(buf + r * 64 + 2 * lane);
                wa[r] = v.x;
                wb[r] = v.y;
            }
        };
        // all 64 walkers active: walk in place, one store
        auto draw_in = [&](uint32_t *buf, uint64_t *bar, uint32_t ph, uint32_t j) {
            mbar_wait(bar, ph);
            uint32_t wa[6], wb[6];
            load(buf, wa, wb);
            gg_walk64x2_r2p(wa, wb, xa, ya, xb, yb);
            const uint64_t idx = (uint64_t)j * a.W + ta - a.g_origin;
            if (V4) {
                *reinterpret_cast<uint4 *>(reinterpret_cast<uint2 *>(a.out) + idx) =
                    make_uint4(xa, ya, xb, yb);
            } else {
                reinterpret_cast<uint2 *>(a.out)[idx] = make_uint2(xa, ya);
                reinterpret_cast<uint2 *>(a.out)[idx + 1] = make_uint2(xb, yb);
            }
            refill(buf, bar, j);
        };
        // edge draws: per-walker range checks
        auto draw_edge = [&](uint32_t *buf, uint64_t *bar, uint32_t ph, uint32_t j) {
            mbar_wait(bar, ph);
            uint32_t wa[6], wb[6];
            load(buf, wa, wb);
            uint32_t nxa = xa, nya = ya, nxb = xb, nyb = yb;
            gg_walk64x2_r2p(wa, wb, nxa, nya, nxb, nyb);
            if (j >= ja0 && j < ja1) {
                xa = nxa;
                ya = nya;
                emit_label<0>(a, (uint64_t)j * a.W + ta - a.g_origin, xa, ya);
            }
            if (j >= jb0 && j < jb1) {
                xb = nxb;
                yb = nyb;
                emit_label<0>(a, (uint64_t)j * a.W + tb - a.g_origin, xb, yb);
            }
            refill(buf, bar, j);
        };
        for (uint32_t j = jlo; j < jhi; j += 2) {
            if (j >= jin0 && j + 2 <= jin1) {  // warp-uniform
                draw_in(buf0, bar0, ph0, j);
                ph0 ^= 1u;
                draw_in(buf1, bar1, ph1, j + 1);
                ph1 ^= 1u;
            } else {
                draw_edge(buf0, bar0, ph0, j);
                ph0 ^= 1u;
                if (j + 1 < jhi) {
                    draw_edge(buf1, bar1, ph1, j + 1);
                    ph1 ^= 1u;
                }
            }
        }
        if (tb < a.W) {
            *reinterpret_cast<uint2 *>(a.x + ta) = make_uint2(xa, xb);
            *reinterpret_cast<uint2 *>(a.y + ta) = make_uint2(ya, yb);
        } else if (ta < a.W) {
            a.x[ta] = xa;
            a.y[ta] = ya;
        }
    }
}

// ---------------------------------------------------------------------------
// Composed-step ("table") walk, l = 64, m = 2^k, forward maps.  The 64 steps
// of a draw are 16 groups of 4 steps; a group reads 12 consecutive record
// bits (fields f0..f3, R3) and the composition of its 4 Gabber-Galil steps
// (§III-A, k = f mod 7, R4) is ONE affine map over Z/2^32:
//     x' = a x + b y + e,   y' = c x + d y + f.
// Every step is affine (sigma_1..3: y += 2x + c; sigma_4..6: x += 2y + c), so
// the composition is exact in wrapped 32-bit arithmetic; over all 4096 bit
// patterns the coefficients are a, d <= 29, b, c <= 22, e, f <= 40 (checked by
// enumeration in tests/test_table_formulation.py), so one 32-bit word holds
// them (5-5-5-5-6-6 bits) and the 4096-entry table is 16 KB of shared memory,
// copied by each block at start from the per-device table in global memory
// (gg::walk_table: forward, then bipartite).  Per group and walker: the 12 bits as a
// scaled table offset (2 ALU), one LDS, the six coefficients (balanced
// between left shifts on the FMA pipe and right shifts on the ALU pipe), four
// IMAD -- ~17 SASS per 4 steps instead of ~25 for four R2P steps.
// ---------------------------------------------------------------------------
constexpr int kTabEntries = 4096;

__device__ __forceinline__ uint32_t gg_compose4(uint32_t p) {
    uint32_t a = 1, b = 0, e = 0, c = 0, d = 1, f = 0;
#pragma unroll
    for (int i = 0; i < 4; i++) {
        const uint32_t k = ((p >> (3 * i)) & 7u) % 7u;
        if (k >= 1 && k <= 3) {  // y <- y + 2x + (k - 1)
            c += 2 * a;
            d += 2 * b;
            f += 2 * e + (k - 1);
        } else if (k >= 4) {     // x <- x + 2y + (k - 4)
            a += 2 * c;
            b += 2 * d;
            e += 2 * f + (k - 4);
        }
    }
    return a | b << 5 | c << 10 | d << 15 | e << 20 | f << 26;
}

// Bipartite variant: a group starts at an even global step
// (l0 even, l = 64), so its steps are sigma, sigma^-1, sigma, sigma^-1; the
// inverse steps subtract (y -= 2x + c | x -= 2y + c) and the composed
// coefficients lie in [-8, 8] (a..d) and [-12, 14] (e, f): the same
// 5-5-5-5-6-6 fields, two's complement, unpacked with arithmetic shifts.
__device__ __forceinline__ uint32_t gg_compose4_bip(uint32_t p) {
    int32_t a = 1, b = 0, e = 0, c = 0, d = 1, f = 0;
#pragma unroll
    for (int i = 0; i < 4; i++) {
        const int32_t k = (int32_t)(((p >> (3 * i)) & 7u) % 7u);
        const int32_t sg = (i & 1) ? -1 : 1;
        if (k >= 1 && k <= 3) {
            c += sg * 2 * a;
            d += sg * 2 * b;
            f += sg * (2 * e + (k - 1));
        } else if (k >= 4) {
            a += sg * 2 * c;
            b += sg * 2 * d;
            e += sg * (2 * f + (k - 4));
        }
    }
    return ((uint32_t)a & 31u) | ((uint32_t)b & 31u) << 5 | ((uint32_t)c & 31u) << 10 |
           ((uint32_t)d & 31u) << 15 | ((uint32_t)e & 63u) << 20 | ((uint32_t)f & 63u) << 26;
}


__global__ void gg_table_init_kernel(uint32_t *tab) {
    const uint32_t p = blockIdx.x * blockDim.x + threadIdx.x;
    if (p < kTabEntries) {
        tab[p] = gg_compose4(p);                    // forward maps
        tab[kTabEntries + p] = gg_compose4_bip(p);  // bipartite variant
    }
}

// Copy a prebuilt table (global memory, 16 KB) into shared memory; the block
// synchronises after.  1024 x 16-byte loads over the block.
__device__ __forceinline__ void gg_stage_table(uint32_t *dst, const uint32_t *src) {
    const uint4 *s4 = reinterpret_cast<const uint4 *>(src);
    uint4 *d4 = reinterpret_cast<uint4 *>(dst);
    for (uint32_t i = threadIdx.x; i < kTabEntries / 4; i += blockDim.x) d4[i] = __ldg(s4 + i);
    __syncthreads();
}

// The table in global memory, once per device (prng_view::tab, staged into
// shared memory by the on-demand consumers).
const uint32_t *walk_table(int device) {
    static std::mutex mu;
    static std::map<int, uint32_t *> tabs;
    std::lock_guard<std::mutex> lk(mu);
    auto it = tabs.find(device);
    if (it != tabs.end()) return it->second;
    uint32_t *t = nullptr;
    if (cudaMalloc(&t, 2 * kTabEntries * 4) != cudaSuccess) return nullptr;
    gg_table_init_kernel<<<kTabEntries / 256, 256>>>(t);
    if (cudaDeviceSynchronize() != cudaSuccess) {
        cudaFree(t);
        return nullptr;
    }
    tabs[device] = t;
    return t;
}

// The pair kernel (adjacent walkers per lane, per-warp TMA, two stages) with
// the composed-step walk; NW warps per block share one table.  EMIT: 0 = u64
// label for m = 2^32 ((y << 32) | x), 1 = u64 label for m = 2^k < 2^32,
// 2 = low u32 word (m <= 2^16); V4: 16-byte stores of two m = 2^32 labels.
// Shared-memory layout.  ORB (table at a 16 KB boundary of the shared
// window, so the group offset ORs into the table base in the masking LOP3
// instead of costing an add per lookup): one raw buffer, the record tiles and
// barriers at its start and the table at the first 16 KB boundary after
// them.  The CTA's shared window begins with a reserved 1 KB, so for the
// buffer at window offset 1 KB the boundary is 15 KB in; the host probes the
// buffer's address once (probe != nullptr: thread 0 reports it and the
// kernel returns) and uses ORB only if the layout fits, else the plain
// layout (table first, added base).
template <int NW>
struct FillTLayout {
    static constexpr uint32_t kTile = 6 * 64;
    static constexpr uint32_t kTileBytes = NW * 2 * kTile * 4;
    static constexpr uint32_t kBarBytes = NW * 2 * 8;
    static constexpr uint32_t kLead = kTileBytes + kBarBytes;   // bytes before the table (ORB)
    static constexpr uint32_t kOrbRaw = 15 * 1024 + kTabEntries * 4;  // ORB buffer
    static constexpr bool kOrbOk = kLead <= 15 * 1024;
};

template <int NW, int EMIT, bool V4, bool BIP = false, bool ORB = false>
__global__ void __launch_bounds__(NW * 32) gg_fill64t_tma_kernel(const __grid_constant__ CUtensorMap tmap,
                                                                 FillArgs a, uint32_t units64,
                                                                 uint32_t *probe) {
    using L = FillTLayout<NW>;
    constexpr int kTile = L::kTile;
    constexpr uint32_t kRaw = ORB ? L::kOrbRaw : kTabEntries * 4 + L::kTileBytes + L::kBarBytes;
    __shared__ __align__(1024) unsigned char raw[kRaw];
    const uint32_t raw_base = (uint32_t)__cvta_generic_to_shared(raw);
    if (probe) {
        if (threadIdx.x == 0 && blockIdx.x == 0) *probe = raw_base;
        return;
    }
    uint32_t tab_off;  // byte offset of the table in raw
    unsigned char *lead;
    if (ORB) {
        tab_off = ((raw_base + 0x3FFFu) & ~0x3FFFu) - raw_base;
        lead = raw;
    } else {
        tab_off = 0;
        lead = raw + kTabEntries * 4;
    }
    uint32_t *tab = reinterpret_cast<uint32_t *>(raw + tab_off);
    auto tiles = reinterpret_cast<uint32_t (*)[2][kTile]>(lead);
    auto bars = reinterpret_cast<uint64_t (*)[2]>(lead + L::kTileBytes);
    const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    uint32_t *buf0 = tiles[wib][0], *buf1 = tiles[wib][1];
    uint64_t *bar0 = &bars[wib][0], *bar1 = &bars[wib][1];
    if (lane == 0) {
        mbar_init(bar0, 1);
        mbar_init(bar1, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    gg_stage_table(tab, a.tab + (BIP ? kTabEntries : 0));  // includes __syncthreads
    const uint32_t tbase = raw_base + tab_off;
    const prng_tab_shifts ksh = prng_tab_shifts_load();
    uint32_t ph0 = 0, ph1 = 0;
    const uint32_t kBytes = kTile * 4;
    for (uint32_t u = warp; u < units64; u += nwarps) {
        const uint32_t ta = u * 64u + 2u * lane, tb = ta + 1u;
        uint32_t ja0 = 0xFFFFFFFFu, ja1 = 0, jb0 = 0xFFFFFFFFu, jb1 = 0;
        if (ta < a.W) {
            walker_draw_range(a.N, a.nl, a.W, ta, ja0, ja1);
            ja0 = max(ja0, a.ja);
            ja1 = min(ja1, a.jb);
        }
        if (tb < a.W) {
            walker_draw_range(a.N, a.nl, a.W, tb, jb0, jb1);
            jb0 = max(jb0, a.ja);
            jb1 = min(jb1, a.jb);
        }
        const uint32_t jlo = __reduce_min_sync(0xFFFFFFFFu, min(ja0, jb0));
        const uint32_t jhi = __reduce_max_sync(0xFFFFFFFFu, max(ja1, jb1));
        if (jlo >= jhi) continue;
        const uint32_t jin0 = __reduce_max_sync(0xFFFFFFFFu, max(ja0, jb0));
        const uint32_t jin1 = __reduce_min_sync(0xFFFFFFFFu, min(ja1, jb1));
        uint32_t xa = 0, ya = 0, xb = 0, yb = 0;
        if (tb < a.W) {
            const uint2 px = *reinterpret_cast<const uint2 *>(a.x + ta);
            const uint2 py = *reinterpret_cast<const uint2 *>(a.y + ta);
            xa = px.x, xb = px.y, ya = py.x, yb = py.y;
        } else if (ta < a.W) {
            xa = a.x[ta];
            ya = a.y[ta];
        }
        if (lane == 0) {
            mbar_expect_tx(bar0, kBytes);
            tma_load_tile(buf0, &tmap, bar0, (int32_t)(u * 64u), (int32_t)((jlo - a.Jw) * 6u));
            if (jlo + 1 < jhi) {
                mbar_expect_tx(bar1, kBytes);
                tma_load_tile(buf1, &tmap, bar1, (int32_t)(u * 64u), (int32_t)((jlo + 1 - a.Jw) * 6u));
            }
        }
        auto refill = [&](uint32_t *buf, uint64_t *bar, uint32_t j) {
            __syncwarp();
            if (lane == 0 && j + 2 < jhi) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                mbar_expect_tx(bar, kBytes);
                tma_load_tile(buf, &tmap, bar, (int32_t)(u * 64u), (int32_t)((j + 2 - a.Jw) * 6u));
            }
        };
        auto load = [&](const uint32_t *buf, uint32_t (&wa)[6], uint32_t (&wb)[6]) {
#pragma unroll
            for (int r = 0; r < 6; r++) {
                const uint2 v = *reinterpret_cast<const uint2 *>(buf + r * 64 + 2 * lane);
                wa[r] = v.x;
                wb[r] = v.y;
            }
        };
        auto draw_in = [&](uint32_t *buf, uint64_t *bar, uint32_t ph, uint32_t j) {
            mbar_wait(bar, ph);
            uint32_t wa[6], wb[6];
            load(buf, wa, wb);
            prng_walk64x2_table_at<BIP, ORB>(tbase, wa, wb, xa, ya, xb, yb, ksh);
            const uint64_t idx = (uint64_t)j * a.W + ta - a.g_origin;
            if (EMIT == 0 && V4) {
                *reinterpret_cast<uint4 *>(reinterpret_cast<uint2 *>(a.out) + idx) =
                    make_uint4(xa, ya, xb, yb);
            } else {
                emit_label<EMIT>(a, idx, xa, ya);
                emit_label<EMIT>(a, idx + 1, xb, yb);
            }
            refill(buf, bar, j);
        };
        auto draw_edge = [&](uint32_t *buf, uint64_t *bar, uint32_t ph, uint32_t j) {
            mbar_wait(bar, ph);
            uint32_t wa[6], wb[6];
            load(buf, wa, wb);
            uint32_t nxa = xa, nya = ya, nxb = xb, nyb = yb;
            prng_walk64x2_table_at<BIP, ORB>(tbase, wa, wb, nxa, nya, nxb, nyb, ksh);
            if (j >= ja0 && j < ja1) {
                xa = nxa;
                ya = nya;
                emit_label<EMIT>(a, (uint64_t)j * a.W + ta - a.g_origin, xa, ya);
            }
            if (j >= jb0 && j < jb1) {
                xb = nxb;
                yb = nyb;
                emit_label<EMIT>(a, (uint64_t)j * a.W + tb - a.g_origin, xb, yb);
            }
            refill(buf, bar, j);
        };
        for (uint32_t j = jlo; j < jhi; j += 2) {
            if (j >= jin0 && j + 2 <= jin1) {  // warp-uniform
                draw_in(buf0, bar0, ph0, j);
                ph0 ^= 1u;
                draw_in(buf1, bar1, ph1, j + 1);
                ph1 ^= 1u;
            } else {
                draw_edge(buf0, bar0, ph0, j);
                ph0 ^= 1u;
                if (j + 1 < jhi) {
                    draw_edge(buf1, bar1, ph1, j + 1);
                    ph1 ^= 1u;
                }
            }
        }
        if (tb < a.W) {
            *reinterpret_cast<uint2 *>(a.x + ta) = make_uint2(xa, xb);
            *reinterpret_cast<uint2 *>(a.y + ta) = make_uint2(ya, yb);
        } else if (ta < a.W) {
            a.x[ta] = xa;
            a.y[ta] = ya;
        }
    }
}

// l = 1 ("emit every vertex"): one 32-bit record word per
// number (R = 1: 3 bits used), so a number costs 4 B read + 8 B written and
// ~10 instructions: the bound is HBM, not the integer pipes.  Each warp owns
// 32 walkers; lane 0 streams 32-draw x 32-walker tiles (4 KB) by TMA into two
// smem stages; lanes step through their column and store coalesced.
constexpr int kL1Draws = 16;

// One l = 1 step for m = 2^k (wrapped): b -> sigma_{b mod 7} (§III-A).
__device__ __forceinline__ void gg_step_l1(uint32_t b, uint32_t &x, uint32_t &y) {
    const uint32_t cy = b - 1u, cx = b - 4u;
    const uint32_t ty = y + 2u * x + cy, tx = x + 2u * y + cx;
    y = (cy < 3u) ? ty : y;
    x = (cx < 3u) ? tx : x;
}

// OST: interior tiles leave through the TMA store engine (the 16 x 32 labels
// staged in shared memory, one cp.async.bulk.tensor store per tile; omap =
// the output as a 2D tensor of 8-byte labels, dim0 = walkers, dim1 = draws)
// instead of 16 STG.64 per lane.
template <int EMIT, int OST = 0>
__global__ void __launch_bounds__(64) gg_fill_l1_tma_kernel(const __grid_constant__ CUtensorMap tmap,
                                                            FillArgs a, uint32_t units,
                                                            const __grid_constant__ CUtensorMap omap) {
    constexpr int kTile = kL1Draws * 32;
    __shared__ __align__(128) uint32_t tiles[kFillWarps][2][kTile];
    __shared__ __align__(128) uint64_t otiles[OST ? kFillWarps : 1][2][OST ? kTile : 1];
    __shared__ __align__(8) uint64_t bars[kFillWarps][2];
    const uint32_t lane = threadIdx.x & 31u, wib = threadIdx.x >> 5;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    uint64_t *bar0 = &bars[wib][0], *bar1 = &bars[wib][1];
    if (lane == 0) {
        mbar_init(bar0, 1);
        mbar_init(bar1, 1);
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncwarp();
    uint32_t ph0 = 0, ph1 = 0;
    const uint32_t kBytes = kTile * 4;
    for (uint32_t u = warp; u < units; u += nwarps) {
        const uint32_t t = u * 32u + lane;
        uint32_t j0 = 0xFFFFFFFFu, j1 = 0;
        if (t < a.W) {
            walker_draw_range(a.N, a.nl, a.W, t, j0, j1);
            j0 = max(j0, a.ja);
            j1 = min(j1, a.jb);
        }
        const uint32_t jlo = __reduce_min_sync(0xFFFFFFFFu, j0);
        const uint32_t jhi = __reduce_max_sync(0xFFFFFFFFu, j1);
        if (jlo >= jhi) continue;
        // A previous unit of this warp (GG_FILL_ONEWAVE / GG_FILL_KPW grids)
        // may have a tile store still reading either output buffer; the
        // in-unit "wait_group.read 1" below only covers stores of this unit
        // (within a unit interior tiles are consecutive, so the newest group
        // always came from the other buffer).
        if (OST && lane == 0) asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
        // draws every lane of the warp emits (empty if some lane is idle)
        const uint32_t jin0 = __reduce_max_sync(0xFFFFFFFFu, j0);
        const uint32_t jin1 = __reduce_min_sync(0xFFFFFFFFu, j1);
        const uint32_t ntiles = (jhi - jlo + kL1Draws - 1) / kL1Draws;
        uint32_t x = 0, y = 0;
        if (t < a.W) {
            x = a.x[t];
            y = a.y[t];
        }
        if (lane == 0) {
            for (uint32_t q = 0; q < 2 && q < ntiles; q++) {
                mbar_expect_tx(&bars[wib][q], kBytes);
                tma_load_tile(tiles[wib][q], &tmap, &bars[wib][q], (int32_t)(u * 32u),
                              (int32_t)(jlo - a.Jw + q * kL1Draws));
            }
        }
        for (uint32_t q = 0; q < ntiles; q++) {
            const uint32_t sidx = q & 1u;
            mbar_wait(&bars[wib][sidx], sidx ? ph1 : ph0);
            if (sidx) ph1 ^= 1u; else ph0 ^= 1u;
            const uint32_t *buf = tiles[wib][sidx];
            const uint32_t jt = jlo + q * kL1Draws;
            if (jt >= jin0 && jt + kL1Draws <= jin1) {
                // interior tile (warp-uniform): all loads first, no per-draw tests
                uint32_t b[kL1Draws];
#pragma unroll
                for (int d = 0; d < kL1Draws; d++) b[d] = buf[d * 32 + lane];
                if (OST) {
                    uint64_t *ob = otiles[OST ? wib : 0][sidx];
                    if (lane == 0)  // the store issued from this buffer two tiles ago has read it
                        asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
                    __syncwarp();
#pragma unroll
                    for (int d = 0; d < kL1Draws; d++) {
                        gg_step_l1(b[d] & 7u, x, y);
                        ob[d * 32 + lane] = EMIT == 0 ? ((uint64_t)y << 32 | x)
                                                      : gg_label(x, y, a.m, a.log2m, true);
                    }
                    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                    __syncwarp();
                    if (lane == 0) {
                        asm volatile(
                            "cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%1, %2}], [%3];"
                            ::"l"(&omap), "r"((int32_t)(u * 32u)), "r"((int32_t)jt),
                              "r"(smem_u32(ob))
                            : "memory");
                        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
                    }
                } else {
                    const uint64_t i0 = (uint64_t)jt * a.W + t - a.g_origin;
#pragma unroll
                    for (int d = 0; d < kL1Draws; d++) {
                        gg_step_l1(b[d] & 7u, x, y);
                        emit_label<EMIT>(a, i0 + (uint64_t)d * a.W, x, y);
                    }
                }
            } else {
#pragma unroll 4
                for (uint32_t d = 0; d < kL1Draws; d++) {
                    const uint32_t j = jt + d;
                    if (j >= j0 && j < j1) {
                        gg_step_l1(buf[d * 32 + lane] & 7u, x, y);
                        emit_label<EMIT>(a, (uint64_t)j * a.W + t - a.g_origin, x, y);
                    }
                }
            }
            __syncwarp();
            if (lane == 0 && q + 2 < ntiles) {
                asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
                mbar_expect_tx(&bars[wib][sidx], kBytes);
                tma_load_tile(tiles[wib][sidx], &tmap, &bars[wib][sidx], (int32_t)(u * 32u),
                              (int32_t)(jt - a.Jw + 2 * kL1Draws));
            }
        }
        if (t < a.W) {
            a.x[t] = x;
            a.y[t] = y;
        }
    }
    if (OST && lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

static PFN_cuTensorMapEncodeTiled_v12000 get_encode() {
    static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
    static bool tried = false;
    if (!tried) {
        tried = true;
        void *p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) ==
                cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            fn = (PFN_cuTensorMapEncodeTiled_v12000)p;
    }
    return fn;
}

// 2D map over the SoA window: dim0 = walkers (pitch), dim1 = rows; box 32 x 6.
// Output of a bulk fill as a 2D tensor of 8-byte labels: element (t, j) at
// out + j * W + t - g_origin; box 32 walkers x kL1Draws draws.  TMA needs a
// 16-byte aligned base and row stride: W even and (out - g_origin) aligned.
static bool make_out_map(CUtensorMap *map, const FillArgs &a) {
    auto enc = get_encode();
    // coordinates are int32: absolute draw indices must stay below 2^31
    if (!enc || (a.W & 1u) || a.jb == 0 || a.jb > 0x7FFFFFF0u) return false;
    const uintptr_t base = (uintptr_t)a.out - (uintptr_t)(a.g_origin * 8ull);
    if (base % 16) return false;
    cuuint64_t dims[2] = {(cuuint64_t)a.W, (cuuint64_t)a.jb};
    cuuint64_t strides[1] = {(cuuint64_t)a.W * 8};
    cuuint32_t box[2] = {32, (cuuint32_t)kL1Draws};
    cuuint32_t estr[2] = {1, 1};
    return enc(map, CU_TENSOR_MAP_DATA_TYPE_UINT64, 2, (void *)base, dims, strides, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
               CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

static bool make_window_map(CUtensorMap *map, const uint32_t *bits, uint64_t pitch, uint64_t rows,
                            uint32_t box_walkers = 32, uint32_t box_rows = 6) {
    auto enc = get_encode();
    if (!enc || rows == 0 || rows > 0x7FFFFFFFull) return false;
    cuuint64_t dims[2] = {(cuuint64_t)pitch, (cuuint64_t)rows};
    cuuint64_t strides[1] = {(cuuint64_t)(pitch * 4)};
    cuuint32_t box[2] = {box_walkers, box_rows};
    cuuint32_t estr[2] = {1, 1};
    CUresult r = enc(map, CU_TENSOR_MAP_DATA_TYPE_UINT32, 2, (void *)bits, dims, strides, box, estr,
                     CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE,
                     CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    return r == CUDA_SUCCESS;
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
            gg_walk_generic(rec, a.pitch, a.l, x, y, (uint32_t)a.m, a.pow2 != 0, a.variant,
                            (uint64_t)a.l0 + (uint64_t)a.l * j);
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

// Any walk length l (2..4096, l != 64), m = 2^k, forward maps: one walker per
// lane, the draw's record read from the window word by word (coalesced across
// the warp) and walked with the R2P step in 10-field groups
// (gg_walk_r2p_any); the generic kernel stays the path for other m and the
// bipartite variant at l != 64.
__global__ void __launch_bounds__(64) gg_fill_any_kernel(FillArgs a, uint32_t units) {
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
            gg_walk_r2p_any(rec, a.pitch, a.l, a.R, x, y);
            const uint64_t lab = gg_label(x, y, a.m, a.log2m, true);
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

// Any walk length with the composed-step table (l != 64, m = 2^k, forward
// maps): the record's 12-bit groups are funnel-shifted out of a rolling pair
// of words (each word loaded once); the last group of a walk whose l is not a
// multiple of 4 masks its unused fields to 0 (sigma_0, stay), so the 4-step
// table also covers 1..3 trailing steps.  4 warps per block share the table.
constexpr int kAnyTW = 4;
__global__ void __launch_bounds__(kAnyTW * 32) gg_fill_anyt_kernel(FillArgs a, uint32_t units) {
    __shared__ __align__(16) uint32_t tab[kTabEntries];
    gg_stage_table(tab, a.tab);
    const uint32_t tbase = (uint32_t)__cvta_generic_to_shared(tab);
    const prng_tab_shifts ksh = prng_tab_shifts_load();
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t warp = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint32_t nwarps = (gridDim.x * blockDim.x) >> 5;
    const uint32_t ngroups = (a.l + 3u) / 4u;
    const uint32_t tail = a.l - 4u * (ngroups - 1u);                 // steps in the last group
    const uint32_t tail_mask = tail >= 4u ? 0xFFFu : ((1u << (3u * tail)) - 1u);
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
            uint32_t lo = __ldg(rec), hi = a.R > 1 ? __ldg(rec + a.pitch) : 0u, wi = 0;
            for (uint32_t g = 0; g < ngroups; g++) {
                const uint32_t bit = 12u * g, i = bit >> 5, sh = bit & 31u;
                if (i != wi) {  // 12-bit groups advance at most one word
                    lo = hi;
                    wi = i;
                    hi = wi + 1 < a.R ? __ldg(rec + (uint64_t)(wi + 1) * a.pitch) : 0u;
                }
                uint32_t idx = __funnelshift_r(lo, hi, sh);
                idx &= (g + 1 == ngroups) ? tail_mask : 0xFFFu;
                prng_group_apply<false>(tbase + 4u * idx, x, y, ksh);
            }
            const uint64_t lab = gg_label(x, y, a.m, a.log2m, true);
            const uint64_t gi = (uint64_t)j * a.W + t;
            if (a.out_u32)
                reinterpret_cast<uint32_t *>(a.out)[gi - a.g_origin] = (uint32_t)lab;
            else
                reinterpret_cast<uint64_t *>(a.out)[gi - a.g_origin] = lab;
        }
        a.x[t] = x;
        a.y[t] = y;
    }
}

// Grid of 64-thread blocks (2 warps each); `units` = work items a warp takes
// round-robin (32 walkers; 64 for the x2 kernels).  One item per warp: the
// block scheduler starts a new block wherever one finishes, so SMs stay busy to
// the end.  A one-wave grid (A/B hook GG_FILL_ONEWAVE=1: as many warps as are
// resident at once, items round-robin) leaves most warps idle during the last
// partial round: C2 (16384 x2 items, 5328 resident warps) 8.15 -> 7.77 ms;
// l = 1 fill (32768 items) 2.56 -> 2.22 ms.
template <class K>
static void plan_grid(K kernel, uint32_t units, int sm_count, uint32_t &blocks, uint32_t &threads) {
    threads = 64;
    blocks = (units + 1) / 2;
    static const bool onewave = getenv("GG_FILL_ONEWAVE") != nullptr;
    if (onewave) {
        int per_sm = 0;
        if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, (int)threads, 0) !=
                cudaSuccess ||
            per_sm <= 0)
            per_sm = 16;
        const uint32_t cap = (uint32_t)sm_count * (uint32_t)per_sm;
        if (blocks > cap) blocks = cap;
    }
    static const int kpw = getenv("GG_FILL_KPW") ? atoi(getenv("GG_FILL_KPW")) : 0;
    if (kpw > 0) {  // experiment: exactly kpw items per warp
        const uint32_t w = (units + kpw - 1) / kpw;
        blocks = (w + 1) / 2;
    }
    if (blocks == 0) blocks = 1;
}

// ORB layout state of the table fill kernel: -1 not probed, 0 plain, 1 ORB.
static int g_orb_state = -1;

void probe_fill_layout(cudaStream_t s) {
    static std::mutex mu;
    std::lock_guard<std::mutex> lk(mu);
    if (g_orb_state >= 0) return;
    g_orb_state = 0;
    if (getenv("GG_FILL_ORB") && atoi(getenv("GG_FILL_ORB")) == 0) return;  // A/B hook
    uint32_t *d = nullptr, hbase = 0;
    if (cudaMalloc(&d, 4) != cudaSuccess) {
        cudaGetLastError();
        return;
    }
    CUtensorMap dummy{};
    FillArgs a{};
    gg_fill64t_tma_kernel<4, 0, true, false, true><<<1, 128, 0, s>>>(dummy, a, 0, d);
    if (cudaMemcpyAsync(&hbase, d, 4, cudaMemcpyDeviceToHost, s) == cudaSuccess &&
        cudaStreamSynchronize(s) == cudaSuccess) {
        const uint32_t off = ((hbase + 0x3FFFu) & ~0x3FFFu) - hbase;
        g_orb_state = (off >= FillTLayout<4>::kLead && off <= 15u * 1024u) ? 1 : 0;
    }
    cudaFree(d);
    cudaGetLastError();  // a failed probe only leaves the plain layout
}

cudaError_t launch_fill(const FillArgs &a, cudaStream_t s, int sm_count) {
    if (a.jb <= a.ja || a.nl == 0) return cudaSuccess;
    const uint32_t units = (a.W + 31u) / 32u;
    uint32_t blocks, threads;
    if (a.l == 1 && a.pow2 && a.variant == 0) {
        CUtensorMap map;
        if (a.rows && make_window_map(&map, a.bits, a.pitch, a.rows, 32, kL1Draws)) {
            CUtensorMap omap;
            static const bool ost_on = !(getenv("GG_L1_TMA_STORE") && atoi(getenv("GG_L1_TMA_STORE")) == 0);
            const bool ost = ost_on && !a.out_u32 && make_out_map(&omap, a);
            if (!ost) memset(&omap, 0, sizeof(omap));
            if (a.out_u32) {
                plan_grid(gg_fill_l1_tma_kernel<2>, units, sm_count, blocks, threads);
                gg_fill_l1_tma_kernel<2><<<blocks, threads, 0, s>>>(map, a, units, omap);
            } else if (a.log2m == 32) {
                if (ost) {
                    plan_grid(gg_fill_l1_tma_kernel<0, 1>, units, sm_count, blocks, threads);
                    gg_fill_l1_tma_kernel<0, 1><<<blocks, threads, 0, s>>>(map, a, units, omap);
                } else {
                    plan_grid(gg_fill_l1_tma_kernel<0>, units, sm_count, blocks, threads);
                    gg_fill_l1_tma_kernel<0><<<blocks, threads, 0, s>>>(map, a, units, omap);
                }
            } else if (ost) {
                plan_grid(gg_fill_l1_tma_kernel<1, 1>, units, sm_count, blocks, threads);
                gg_fill_l1_tma_kernel<1, 1><<<blocks, threads, 0, s>>>(map, a, units, omap);
            } else {
                plan_grid(gg_fill_l1_tma_kernel<1>, units, sm_count, blocks, threads);
                gg_fill_l1_tma_kernel<1><<<blocks, threads, 0, s>>>(map, a, units, omap);
            }
            return cudaGetLastError();
        }
    }
    // composed-step table walk (the default for l = 64, m = 2^k, forward maps);
    // GG_FILL_TABLE = warps per block (2, 4, 8; default 4: 63 registers, 7 blocks
    // = 28 warps per SM, shared memory bound; C2 A/B 4.78 / 5.01 / 5.22 ms for
    // 4 / 8 / 2, 5.08 ms for 8 warps at 48 registers), 0 = the R2P kernels
    static const int table_nw = getenv("GG_FILL_TABLE") ? atoi(getenv("GG_FILL_TABLE")) : 4;
    // ORB layout (table at a 16 KB boundary, FillTLayout), probed by
    // probe_fill_layout at handle creation; plain layout until then
    const bool orb = g_orb_state == 1;
    if (a.l == 64 && a.pow2 && a.variant == 1 && (a.l0 & 1u) == 0 && table_nw > 0 && a.rows &&
        getenv("GG_FILL_NO_BIP") == nullptr) {
        // bipartite variant: the signed composed-step table (4 warps per block)
        CUtensorMap map;
        const uint32_t units64 = (a.W + 63u) / 64u;
        if (make_window_map(&map, a.bits, a.pitch, a.rows, 64)) {
            const uint32_t blocks = (units64 + 3) / 4;
#define GG_LAUNCH_B(E, O)                                                                         \
    gg_fill64t_tma_kernel<4, E, false, true, O><<<blocks, 128, 0, s>>>(map, a, units64, nullptr)
            if (a.out_u32) { if (orb) GG_LAUNCH_B(2, true); else GG_LAUNCH_B(2, false); }
            else if (a.log2m != 32) { if (orb) GG_LAUNCH_B(1, true); else GG_LAUNCH_B(1, false); }
            else { if (orb) GG_LAUNCH_B(0, true); else GG_LAUNCH_B(0, false); }
#undef GG_LAUNCH_B
            return cudaGetLastError();
        }
    }
    if (a.l == 64 && a.pow2 && a.variant == 0 && table_nw > 0 && a.rows) {
        CUtensorMap map;
        const uint32_t units64 = (a.W + 63u) / 64u;
        if (make_window_map(&map, a.bits, a.pitch, a.rows, 64)) {
            const bool v4 = (a.W % 2 == 0) && (a.g_origin % 2 == 0) && ((uintptr_t)a.out % 16 == 0);
            // one 64-walker unit per warp; A/B hook GG_FILL_KPW = units per warp
            static const int kpw_t = getenv("GG_FILL_KPW") ? std::max(1, atoi(getenv("GG_FILL_KPW"))) : 1;
#define GG_LAUNCH_T(NW, E, V, O)                                                                  \
    gg_fill64t_tma_kernel<NW, E, V, false, O>                                                     \
        <<<(units64 + NW * kpw_t - 1) / (NW * kpw_t), NW * 32, 0, s>>>(map, a, units64, nullptr)
#define GG_LAUNCH_TNW(NW, O)                                                                      \
    do {                                                                                          \
        if (a.out_u32) GG_LAUNCH_T(NW, 2, false, O);                                              \
        else if (a.log2m != 32) GG_LAUNCH_T(NW, 1, false, O);                                     \
        else if (v4) GG_LAUNCH_T(NW, 0, true, O);                                                 \
        else GG_LAUNCH_T(NW, 0, false, O);                                                        \
    } while (0)
            if (table_nw >= 8) GG_LAUNCH_TNW(8, false);  // 8 warps' tiles exceed the ORB lead
            else if (table_nw >= 4) { if (orb) GG_LAUNCH_TNW(4, true); else GG_LAUNCH_TNW(4, false); }
            else { if (orb) GG_LAUNCH_TNW(2, true); else GG_LAUNCH_TNW(2, false); }
#undef GG_LAUNCH_TNW
#undef GG_LAUNCH_T
            return cudaGetLastError();
        }
    }
    if (a.l == 64 && a.pow2 && a.variant == 1 && (a.l0 & 1u) == 0 && a.rows &&
        getenv("GG_FILL_NO_BIP") == nullptr) {
        // bipartite variant (f1): every draw starts at an even global step
        // (l0 + 64 j), so the fixed (sigma, sigma^-1) pairing of the R2P walk holds
        CUtensorMap map;
        const uint32_t units64 = (a.W + 63u) / 64u;
        if (make_window_map(&map, a.bits, a.pitch, a.rows, 64)) {
            if (a.out_u32) {
                plan_grid(gg_fill64x2_tma_kernel<2, 1, 1, 1, true>, units64, sm_count, blocks, threads);
                gg_fill64x2_tma_kernel<2, 1, 1, 1, true><<<blocks, threads, 0, s>>>(map, a, units64);
            } else if (a.log2m == 32) {
                plan_grid(gg_fill64x2_tma_kernel<0, 1, 1, 1, true>, units64, sm_count, blocks, threads);
                gg_fill64x2_tma_kernel<0, 1, 1, 1, true><<<blocks, threads, 0, s>>>(map, a, units64);
            } else {
                plan_grid(gg_fill64x2_tma_kernel<1, 1, 1, 1, true>, units64, sm_count, blocks, threads);
                gg_fill64x2_tma_kernel<1, 1, 1, 1, true><<<blocks, threads, 0, s>>>(map, a, units64);
            }
            return cudaGetLastError();
        }
    }
    if (a.l == 64 && !a.pow2 && a.variant == 0 && a.m <= (1ull << 30) && a.rows &&
        getenv("GG_FILL_NO_MOD") == nullptr) {
        // other m <= 2^30: the R2P step with two conditional subtracts per step
        CUtensorMap map;
        const uint32_t units64 = (a.W + 63u) / 64u;
        if (make_window_map(&map, a.bits, a.pitch, a.rows, 64)) {
            if (a.out_u32) {
                plan_grid(gg_fill64x2_tma_kernel<4, 1, 1, 1, false, true>, units64, sm_count, blocks, threads);
                gg_fill64x2_tma_kernel<4, 1, 1, 1, false, true><<<blocks, threads, 0, s>>>(map, a, units64);
            } else {
                plan_grid(gg_fill64x2_tma_kernel<3, 1, 1, 1, false, true>, units64, sm_count, blocks, threads);
                gg_fill64x2_tma_kernel<3, 1, 1, 1, false, true><<<blocks, threads, 0, s>>>(map, a, units64);
            }
            return cudaGetLastError();
        }
    }
    if (a.l == 64 && a.pow2 && a.variant == 0) {
        CUtensorMap map;
        static const bool use_tma = getenv("GG_FILL_NO_TMA") == nullptr;
        static const bool use_x2 = getenv("GG_FILL_X1") == nullptr;
        const uint32_t units64 = (a.W + 63u) / 64u;
        if (use_tma && use_x2 && a.rows && make_window_map(&map, a.bits, a.pitch, a.rows, 64)) {
            if (a.out_u32) {
                plan_grid(gg_fill64x2_tma_kernel<2>, units64, sm_count, blocks, threads);
                gg_fill64x2_tma_kernel<2><<<blocks, threads, 0, s>>>(map, a, units64);
            } else if (a.log2m == 32) {
                // A/B hooks (measured on B200, C2 fill, profiles/r01_*):
                //   GG_FILL_STEP=0  per-step LOP3.P predicates instead of R2P (8.93 vs 8.13 ms)
                //   GG_FILL_U2=0    one draw per loop iteration instead of two (8.17 vs 8.13)
                //   GG_FILL_MINB=24 37-40 registers / 48 warps per SM instead of ptxas' 55 /
                //                   36 warps (8.39 vs 8.13: the R2P step wants the registers)
                static const int minb = getenv("GG_FILL_MINB") ? atoi(getenv("GG_FILL_MINB")) : 1;
                static const bool r2p = !(getenv("GG_FILL_STEP") && atoi(getenv("GG_FILL_STEP")) == 0);
                static const bool u2 = !(getenv("GG_FILL_U2") && atoi(getenv("GG_FILL_U2")) == 0);
                static const bool pair = getenv("GG_FILL_PAIR") && atoi(getenv("GG_FILL_PAIR")) == 1;
                if (pair && r2p && minb == 1 && u2) {
                    // adjacent-walker lanes (LDS.64, 16-B stores when the output index parity allows)
                    const bool v4 = (a.W % 2 == 0) && (a.g_origin % 2 == 0) &&
                                    ((uintptr_t)a.out % 16 == 0);
                    if (v4) {
                        plan_grid(gg_fill64p_tma_kernel<true>, units64, sm_count, blocks, threads);
                        gg_fill64p_tma_kernel<true><<<blocks, threads, 0, s>>>(map, a, units64);
                    } else {
                        plan_grid(gg_fill64p_tma_kernel<false>, units64, sm_count, blocks, threads);
                        gg_fill64p_tma_kernel<false><<<blocks, threads, 0, s>>>(map, a, units64);
                    }
                    return cudaGetLastError();
                }
#define GG_LAUNCH_X2(...)                                                                   \
    do {                                                                                    \
        plan_grid(gg_fill64x2_tma_kernel<__VA_ARGS__>, units64, sm_count, blocks, threads); \
        gg_fill64x2_tma_kernel<__VA_ARGS__><<<blocks, threads, 0, s>>>(map, a, units64);    \
    } while (0)
                if (!r2p)
                    GG_LAUNCH_X2(0, 24, 0, 0);
                else if (minb == 24 && !u2)
                    GG_LAUNCH_X2(0, 24, 1, 0);
                else if (minb == 24)
                    GG_LAUNCH_X2(0, 24, 1, 1);
                else if (!u2)
                    GG_LAUNCH_X2(0, 1, 1, 0);
                else
                    GG_LAUNCH_X2(0, 1, 1, 1);
#undef GG_LAUNCH_X2
            } else {
                plan_grid(gg_fill64x2_tma_kernel<1>, units64, sm_count, blocks, threads);
                gg_fill64x2_tma_kernel<1><<<blocks, threads, 0, s>>>(map, a, units64);
            }
        } else if (use_tma && a.rows && make_window_map(&map, a.bits, a.pitch, a.rows)) {
            if (a.out_u32) {
                plan_grid(gg_fill64_tma_kernel<2>, units, sm_count, blocks, threads);
                gg_fill64_tma_kernel<2><<<blocks, threads, 0, s>>>(map, a, units);
            } else if (a.log2m == 32) {
                plan_grid(gg_fill64_tma_kernel<0>, units, sm_count, blocks, threads);
                gg_fill64_tma_kernel<0><<<blocks, threads, 0, s>>>(map, a, units);
            } else {
                plan_grid(gg_fill64_tma_kernel<1>, units, sm_count, blocks, threads);
                gg_fill64_tma_kernel<1><<<blocks, threads, 0, s>>>(map, a, units);
            }
        } else if (a.out_u32) {
            plan_grid(gg_fill64_kernel<1>, units, sm_count, blocks, threads);
            gg_fill64_kernel<1><<<blocks, threads, 0, s>>>(a, units);
        } else {
            plan_grid(gg_fill64_kernel<0>, units, sm_count, blocks, threads);
            gg_fill64_kernel<0><<<blocks, threads, 0, s>>>(a, units);
        }
    } else if (a.pow2 && a.variant == 0 && a.l >= 2 && getenv("GG_FILL_NO_ANY") == nullptr) {
        if (table_nw > 0) {
            // composed-step table; GG_FILL_TABLE=0: the R2P any-l kernel
            gg_fill_anyt_kernel<<<(units + kAnyTW - 1) / kAnyTW, kAnyTW * 32, 0, s>>>(a, units);
        } else {
            plan_grid(gg_fill_any_kernel, units, sm_count, blocks, threads);
            gg_fill_any_kernel<<<blocks, threads, 0, s>>>(a, units);
        }
    } else {
        plan_grid(gg_fill_generic_kernel, units, sm_count, blocks, threads);
        gg_fill_generic_kernel<<<blocks, threads, 0, s>>>(a, units);
    }
    return cudaGetLastError();
}

}  // namespace gg

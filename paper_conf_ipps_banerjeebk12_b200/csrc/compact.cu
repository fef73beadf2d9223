// Stable stream compaction in one pass (decoupled look-back), used by the
// on-demand consumers between epochs:
//   list ranking (§V Alg.3 l.10): after a round of ReduceList the
//     survivors stay in order (reading R16: walker i serves active slot i, so
//     slot order is part of the result) and the removed nodes go to the
//     re-insertion log; Phase II keeps the splitters;
//   Monte Carlo (§VI Alg.4): the threads that still have photons form
//     the next epoch's walker list.
//
// One CTA per tile of kTile = 256 threads x 8 items, tiles taken in launch
// order through an atomic ticket (so every tile's predecessors are running
// or done: the look-back cannot deadlock).  Each tile publishes its kept
// count (flag AGG), then adds its predecessors' counts walking back until it
// meets an inclusive prefix (flag INC), and publishes its own inclusive
// prefix.  Per tile: items striped over the threads (coalesced 4-B loads),
// per row a warp ballot gives each item's rank among the kept items of its
// warp row; one warp scans the 8 x 8 (row, warp) counts in row-major order.
//
// Traffic per item: 1 B flag + 4 B index read (none when the input is the
// identity), 4 B written; per tile one 8-B status word and a few look-back
// reads.  HBM-bound; the per-round launch is a few microseconds at 2^24.
#include <cstdint>

#include <cuda_runtime.h>

#include "gg_internal.h"

namespace {

constexpr int kThreads = 256;
constexpr int kItems = 8;
constexpr int kTile = kThreads * kItems;
constexpr int kWarps = kThreads / 32;
constexpr uint64_t kFlagAgg = 1ull << 62, kFlagInc = 2ull << 62;
constexpr uint64_t kValueMask = (1ull << 62) - 1;

__device__ __forceinline__ uint64_t load_status(const uint64_t *p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}

__device__ __forceinline__ void store_status(uint64_t *p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}

__global__ void __launch_bounds__(kThreads) compact_kernel(const int32_t *in, const uint8_t *flags,
                                                           int64_t n, int32_t *kept_out,
                                                           int32_t *removed_out,
                                                           int32_t *d_count,
                                                           volatile uint64_t *h_count,
                                                           uint32_t tag, uint64_t *status,
                                                           uint32_t *ticket, uint32_t ntiles) {
    __shared__ uint32_t s_tile;
    __shared__ uint32_t s_cnt[kItems][kWarps];  // kept per (row, warp), then exclusive offsets
    __shared__ uint64_t s_excl;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) s_tile = atomicAdd(ticket, 1u);
    __syncthreads();
    const uint32_t tile = s_tile;
    const int64_t base = (int64_t)tile * kTile;
    bool keep[kItems];
    int32_t val[kItems];
#pragma unroll
    for (int k = 0; k < kItems; k++) {
        const int64_t i = base + k * kThreads + threadIdx.x;
        keep[k] = false;
        val[k] = 0;
        if (i < n) {
            keep[k] = flags[i] != 0;
            val[k] = in ? in[i] : (int32_t)i;
        }
    }
    uint32_t rank_in_row[kItems];
#pragma unroll
    for (int k = 0; k < kItems; k++) {
        const uint32_t b = __ballot_sync(0xFFFFFFFFu, keep[k]);
        rank_in_row[k] = __popc(b & ((1u << lane) - 1u));
        if (lane == 0) s_cnt[k][warp] = __popc(b);
    }
    __syncthreads();
    if (warp == 0) {
        // exclusive scan of the 64 (row, warp) counts in row-major order:
        // lane holds entries 2*lane, 2*lane + 1
        const uint32_t *flat = &s_cnt[0][0];
        const uint32_t a = flat[2 * lane], b = flat[2 * lane + 1];
        uint32_t incl = a + b;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint32_t t = __shfl_up_sync(0xFFFFFFFFu, incl, o);
            if (lane >= o) incl += t;
        }
        const uint32_t excl = incl - a - b;
        const uint32_t total = __shfl_sync(0xFFFFFFFFu, incl, 31);
        __syncwarp();
        uint32_t *w = &s_cnt[0][0];
        w[2 * lane] = excl;
        w[2 * lane + 1] = excl + a;
        if (lane == 0) {
            // publish, then look back over the predecessors
            uint64_t excl_tile = 0;
            if (tile == 0) {
                store_status(&status[0], kFlagInc | total);
            } else {
                store_status(&status[tile], kFlagAgg | total);
                for (int64_t j = (int64_t)tile - 1; j >= 0;) {
                    const uint64_t st = load_status(&status[j]);
                    if (st & kFlagInc) {
                        excl_tile += st & kValueMask;
                        break;
                    }
                    if (st & kFlagAgg) {
                        excl_tile += st & kValueMask;
                        j--;
                    }
                    // else: predecessor not published yet; spin
                }
                store_status(&status[tile], kFlagInc | (excl_tile + total));
            }
            s_excl = excl_tile;
            if (tile == ntiles - 1) {
                *d_count = (int32_t)(excl_tile + total);
                if (h_count) {
                    __threadfence_system();
                    *h_count = ((uint64_t)tag << 32) | (uint32_t)(excl_tile + total);
                }
            }
        }
    }
    __syncthreads();
    const int64_t kept_before = (int64_t)s_excl;
#pragma unroll
    for (int k = 0; k < kItems; k++) {
        const int64_t i = base + k * kThreads + threadIdx.x;
        if (i >= n) continue;
        const int64_t r = (int64_t)s_cnt[k][warp] + rank_in_row[k];  // kept before i in the tile
        if (keep[k]) {
            kept_out[kept_before + r] = val[k];
        } else if (removed_out) {
            const int64_t pos_in_tile = k * kThreads + threadIdx.x;
            removed_out[(base - kept_before) + (pos_in_tile - r)] = val[k];
        }
    }
}

}  // namespace

size_t gg::compact_scratch_bytes(int64_t n) {
    const int64_t tiles = (n + kTile - 1) / kTile;
    return (size_t)(tiles + 1) * 8;
}

cudaError_t gg::compact_flagged(const int32_t *in, const uint8_t *flags, int64_t n,
                                int32_t *kept_out, int32_t *removed_out, int32_t *d_count,
                                volatile uint64_t *h_count, uint32_t tag, void *scratch,
                                cudaStream_t s) {
    if (n <= 0) {
        cudaError_t e = cudaMemsetAsync(d_count, 0, 4, s);
        if (e == cudaSuccess && h_count) *h_count = (uint64_t)tag << 32;
        return e;
    }
    const uint32_t tiles = (uint32_t)((n + kTile - 1) / kTile);
    uint64_t *status = (uint64_t *)scratch;
    uint32_t *ticket = (uint32_t *)(status + tiles);
    cudaError_t e = cudaMemsetAsync(scratch, 0, compact_scratch_bytes(n), s);
    if (e != cudaSuccess) return e;
    compact_kernel<<<tiles, kThreads, 0, s>>>(in, flags, n, kept_out, removed_out, d_count, h_count,
                                              tag, status, ticket, tiles);
    return cudaGetLastError();
}

// Synthetic on-demand consumer (include/gg_apps.h: gg_consume): every
// thread owns one walker and calls the header-only prng_next
// (prng_device.cuh) a data-dependent number of times — the usage pattern of
// Alg.3 l.6 and Alg.4 l.3 without the application around it.
#include <cstdint>

#include <cuda_runtime.h>

#include "gg_apps.h"
#include "prng.h"
#include "prng_device.cuh"

namespace {

// MODE: the walk compiled into this instantiation (prng_walk_mode of the
// view, picked on the host), so the hot loop holds one walk, not the
// run-time dispatch over all of them.
template <int MODE>
__global__ void __launch_bounds__(128) consume_kernel(const __grid_constant__ prng_view v,
                                                      uint64_t threads,
                                                      const uint32_t *counts, uint32_t uniform,
                                                      uint64_t *out, const uint64_t *offsets,
                                                      uint64_t *xor_out) {
    // the paper's generator (PRNG_WALK_L64): composed-step table in shared
    // memory -- staged only by blocks where some thread makes >= kTabMin
    // draws (16 KB of staging for a block of one-draw threads costs more
    // than it saves: the list-ranking-shaped consumers)
    constexpr bool TAB_MODE = MODE == PRNG_WALK_L64;
    constexpr uint32_t kTabMin = 4;
    __shared__ __align__(PRNG_TABLE_ALIGN) uint32_t tab[TAB_MODE ? PRNG_TABLE_WORDS : 4];
    const uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
    const uint32_t c = t < threads ? (counts ? counts[t] : uniform) : 0u;
    bool TAB = false;
    if (TAB_MODE) {
        TAB = __syncthreads_or(c >= kTabMin) != 0;  // block-uniform
        if (TAB) {
            prng_table_stage(&v, tab);
            __syncthreads();
        }
    }
    if (t >= threads) return;
    if (c == 0) {  // idle this launch: the walker's state is untouched
        if (xor_out) xor_out[t] = 0;
        return;
    }
    prng_state st = prng_state_load(&v, (uint32_t)t);
    uint64_t acc = 0;
    const uint64_t base = out ? (offsets ? offsets[t] : t * (uint64_t)uniform) : 0;
    uint32_t r = 0;
    for (; r + 4 <= c; r += 4) {  // four records' loads in flight together
        uint64_t z4[4];
        if (TAB)
            prng_next_n_table<4>(&st, &v, tab, z4);
        else
            prng_next_n<4, false, MODE>(&st, &v, z4);
#pragma unroll
        for (int k = 0; k < 4; k++) {
            acc ^= z4[k];
            if (out) out[base + r + k] = z4[k];
        }
    }
    for (; r < c; r++) {
        const uint64_t z = TAB ? prng_next_table(&st, &v, tab) : prng_next<MODE>(&st, &v);
        acc ^= z;
        if (out) out[base + r] = z;
    }
    prng_state_store(&v, &st);
    if (xor_out) xor_out[t] = acc;
}

}  // namespace

extern "C" int gg_consume(prng_t *h, uint64_t threads, const uint32_t *counts, uint32_t uniform,
                          uint64_t *out, const uint64_t *offsets, uint64_t *xor_out,
                          void *stream) {
    if (!h) return PRNG_E_INVALID;
    prng_view v;
    int rc = prng_device_view(h, &v, sizeof(v));
    if (rc != PRNG_OK) return rc;
    if (threads == 0) return PRNG_OK;
    if (threads > v.Wv) return PRNG_E_INVALID;
    auto mis = [](const void *p, uintptr_t a) { return p && ((uintptr_t)p % a) != 0; };
    if (mis(counts, 4) || mis(out, 8) || mis(offsets, 8) || mis(xor_out, 8)) return PRNG_E_INVALID;
    const uint32_t tpb = 128;
    const uint64_t blocks = (threads + tpb - 1) / tpb;
    cudaStream_t st = (cudaStream_t)stream;
#define GG_CONSUME(M)                                                                        \
    consume_kernel<M><<<(unsigned)blocks, tpb, 0, st>>>(v, threads, counts, uniform, out, offsets, \
                                                        xor_out)
    switch (prng_walk_mode(&v)) {
    case PRNG_WALK_L64: GG_CONSUME(PRNG_WALK_L64); break;
    case PRNG_WALK_L64_BIP: GG_CONSUME(PRNG_WALK_L64_BIP); break;
    case PRNG_WALK_ANY_POW2: GG_CONSUME(PRNG_WALK_ANY_POW2); break;
    case PRNG_WALK_L64_MOD: GG_CONSUME(PRNG_WALK_L64_MOD); break;
    default: GG_CONSUME(PRNG_WALK_GENERIC); break;
    }
#undef GG_CONSUME
    return cudaGetLastError() == cudaSuccess ? PRNG_OK : PRNG_E_CUDA;
}

/*
 * include/gg_apps.h — C ABI of the on-demand consumers of the expander-walk
 * PRNG (§V list ranking and §VI Monte Carlo) and of the
 * synthetic on-demand demand generator used for measurement.
 *
 * Same conventions as prng.h: plain C types, int status (PRNG_* codes),
 * caller-owned buffers, `stream` = cudaStream_t as void*, device pointers
 * on the handle's device.  Each entry point runs entirely in the library's
 * CUDA kernels; the prng_t handle supplies the bits (FEED/TRANSFER) and the
 * walker state.
 */
#ifndef GGPRNG_GG_APPS_H
#define GGPRNG_GG_APPS_H

#include <stddef.h>
#include <stdint.h>

#include "prng.h"

#ifdef __cplusplus
extern "C" {
#endif

/*
 * Synthetic on-demand consumer (GetNextRand called from user threads,
 * P:12 §III "any thread of the GPU can make a request ... at any point of
 * time"; Alg.2).  Inside an open epoch (prng_epoch_begin), thread t of
 * a grid of `threads` threads uses walker t and calls prng_next
 * counts[t] times (counts == NULL: `uniform` times).
 *   out     : if non-NULL, the r-th number of thread t is written to
 *             out[offsets[t] + r] (offsets == NULL: t * uniform + r).
 *   xor_out : if non-NULL, thread t writes the XOR of its numbers to
 *             xor_out[t] (used for throughput runs: 8 B per thread).
 * Numbers past the window return 0 and set the overrun flag (prng_check).
 * All pointers are device pointers; counts/offsets may be NULL.
 */
int gg_consume(prng_t *h, uint64_t threads, const uint32_t *counts, uint32_t uniform,
               uint64_t *out, const uint64_t *offsets, uint64_t *xor_out, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* GGPRNG_GG_APPS_H */

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

/*
 * Randomised list ranking (§V): rank[v] = distance of node v
 * from the head (R17), computed by Alg.3 ReduceList (FIS rounds with
 * on-demand draws), Helman-JaJa [10] splitter ranking of the reduced
 * list, and re-insertion of the removed nodes ("the nodes removed in
 * step 1 are re-inserted to get the final ranks").
 *   h             : generator with at least n walkers, no epoch open.  The
 *                   call opens one on-demand epoch per Phase I round (the
 *                   active count is only known after the previous round) and
 *                   one for the splitter choice; walker i serves the node in
 *                   active slot i (R16').
 *   n             : list size, 1 <= n <= 2^24.
 *   succ, pred    : device int32[n]: successor / predecessor (-1 at the
 *                   tail / head); not modified.  head: index of the head.
 *   rank          : device int32[n], output.
 *   removed_round : optional device int32[n]: Phase I round in which the node
 *                   was removed, -1 if it stayed (for parity checks).
 *   is_splitter   : optional device int32[n]: 1 for Phase II splitters.
 *   info          : optional HOST int64[8]: rounds, reduced size, splitters,
 *                   draws, Phase I / II / III device microseconds, rounds.
 * Synchronous (returns when rank is final).  Temporary device memory is
 * stream-ordered (cudaMallocAsync) on `stream`.
 */
int gg_list_rank(prng_t *h, int64_t n, const int32_t *succ, const int32_t *pred, int64_t head,
                 int32_t *rank, int32_t *removed_round, int32_t *is_splitter, int64_t *info,
                 void *stream);

#ifdef __cplusplus
}
#endif
#endif /* GGPRNG_GG_APPS_H */

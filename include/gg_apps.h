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
 * Collectives supplied by the caller for multi-GPU runs (one process per
 * GPU).  The library stays independent of any communication runtime: the
 * Python layer implements these with torch.distributed (NCCL over
 * NVLink/NVSwitch on the GPU box, gloo in tests).  Buffers are DEVICE
 * pointers of the calling rank's GPU; each call is synchronous with respect
 * to the device work enqueued before it (the library synchronises its
 * stream first) and returns 0 on success.
 *   allgather     : recv[r * bytes + i] = send_of_rank_r[i], i < bytes
 *   allreduce_i32 : buf[i] = sum over ranks of buf_of_rank[i], i < count
 */
typedef int (*gg_allgather_fn)(void *ctx, const void *send, void *recv, size_t bytes);
typedef int (*gg_allreduce_i32_fn)(void *ctx, int32_t *buf, size_t count);
typedef struct {
    int rank, world;
    gg_allgather_fn allgather;
    gg_allreduce_i32_fn allreduce_i32;
    void *ctx;
} gg_collective;

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
 *   coll          : NULL for one GPU.  With world > 1 every rank calls with the
 *                   same list and a generator of the same seed and walker ids:
 *                   Phase I is replicated (it is deterministic), Phase II walks
 *                   only this rank's share of the splitters' sublists, the
 *                   splitter records (sublist length, next splitter) are
 *                   exchanged with one allgather (the north star's "splitter
 *                   exchange"), the prefix over splitters is computed on every
 *                   rank, the reduced-list ranks are combined with one int32
 *                   allreduce, and Phase III runs replicated; every rank ends
 *                   with the full rank array.
 * Synchronous (returns when rank is final).  Temporary device memory is
 * stream-ordered (cudaMallocAsync) on `stream`.
 */
int gg_list_rank(prng_t *h, int64_t n, const int32_t *succ, const int32_t *pred, int64_t head,
                 int32_t *rank, int32_t *removed_round, int32_t *is_splitter, int64_t *info,
                 const gg_collective *coll, void *stream);

/* ---------------------------------------------------------------------------
 * Monte Carlo photon migration (§VI, Alg.4): photons from a
 * pencil beam at the origin travel through a stack of layers; at every
 * interaction a fraction mua/(mua+mus) of the weight is absorbed and the
 * packet is scattered (Henyey-Greenstein); packets below the weight
 * threshold are terminated; boundaries reflect/refract by Fresnel's law.
 * Weights are drawn on demand with prng_next (Alg.4 l.3), as are step
 * lengths, scattering angles and Fresnel decisions.  Readings R19-R22 in
 * DESIGN.md §3 fix what the paper leaves open (draw order, fixed point).
 * ------------------------------------------------------------------------- */
#define GG_MC_MAX_LAYERS 16
#define GG_MC_TALLY_FIXED 5

typedef struct {
    double n;    /* refractive index */
    double mua;  /* absorption coefficient [1/cm] */
    double mus;  /* scattering coefficient [1/cm] */
    double g;    /* Henyey-Greenstein anisotropy, (-1, 1) */
    double d;    /* thickness [cm], > 0 */
} gg_mc_layer;

typedef struct {
    const gg_mc_layer *layers;  /* host array of nlayers (1..GG_MC_MAX_LAYERS) */
    int nlayers;
    double n_top, n_bottom;     /* ambient refractive indices above / below */
    uint64_t photons_total;     /* P over all shards */
    uint64_t threads_total;     /* global GPU threads over all shards */
    uint64_t thread0;           /* global id of this call's thread 0 (= walker_base) */
    uint64_t threads;           /* threads of this call; walker i serves thread i */
    uint32_t epoch_draws;       /* D = 3K draws per walker per epoch, multiple of 3 */
    double w_threshold;         /* terminate below this weight (1e-4) */
} gg_mc_config;

/*
 * Run the simulation for global threads [thread0, thread0 + threads); thread
 * tg simulates P/Tg photons (+1 if tg < P mod Tg), so shards over GPUs sum to
 * the single-GPU result exactly.
 *   tallies    : HOST int64[GG_MC_TALLY_FIXED + nlayers], ADDED to, weight
 *                units 2^-32: launched, specular, diffuse reflectance R_d,
 *                transmittance T_t, terminated, absorbed per layer.
 *                launched = sum of the others exactly.
 *   per_thread : optional DEVICE int64[threads * (5 + nlayers)] (parity checks).
 *   stats      : optional HOST int64[7]: photons, draws, epochs,
 *                interactions, kernel microseconds, total microseconds,
 *                walker-epochs fed (each = D draws of host bits).  Each
 *                epoch's window holds only the threads that still had work
 *                one epoch earlier (prng_epoch_begin_list), fed while the
 *                previous epoch's kernel runs.
 * Synchronous.  The handle needs >= threads walkers and no open epoch.
 */
int gg_mc_run(prng_t *h, const gg_mc_config *cfg, int64_t *tallies, int64_t *per_thread,
              int64_t *stats, void *stream);

#ifdef __cplusplus
}
#endif
#endif /* GGPRNG_GG_APPS_H */

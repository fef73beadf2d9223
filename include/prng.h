/*
 * include/prng.h — C ABI of the B200 expander-walk PRNG.
 *
 * Method: Banerjee, Bahl & Kothapalli, "An On-Demand Fast Parallel Pseudo
 * Random Number Generator with Applications", IPDPS Workshops 2012
 * (/root/reference/PAPER.md; "P:14 §III-B Alg.1" = PAPER.md line 14 = PDF
 * page 3, section III-B, Algorithm 1).  Readings R1..R22 of passages the
 * paper leaves silent or garbled are listed in DESIGN.md §3.
 *
 * Every walker performs a random walk on the implicit 7-regular Gabber–Galil
 * expander on Z_m x Z_m (§III-A); each step consumes 3 bits of a
 * host-supplied seed-bit stream ("it requires only 3 bits"); after
 * Alg.1's 64-step burn-in every further walk of l = 64 steps yields the
 * walker's vertex label as one 64-bit random number (Alg.2).
 *
 * Conventions for every call:
 *   - Plain C types only.  Device pointers are CUDA device addresses of the
 *     handle's device; `stream` is a cudaStream_t passed as void* (NULL =
 *     legacy default stream).
 *   - Every call returns an int status (PRNG_OK = 0 or a negative PRNG_E_*).
 *     Invalid arguments return PRNG_E_INVALID with no side effects.  A CUDA
 *     failure returns PRNG_E_CUDA and poisons the handle: later calls return
 *     PRNG_E_STATE until prng_destroy.
 *   - The library owns walker state, bit windows, pinned host slots, feed
 *     threads, its own streams and events.  The caller owns every buffer it
 *     passes in.  No exception crosses the ABI.
 *   - One host thread at a time per handle.  Device side: any number of GPU
 *     threads may call prng_next (prng_device.cuh), each on its own walker.
 *   - Determinism contract: every number is a pure function of (graph
 *     params, seed, global walker id, draw index) — independent of launch
 *     geometry, epoch depth, host thread count, GPU count and call chunking.
 */
#ifndef GGPRNG_PRNG_H
#define GGPRNG_PRNG_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct prng_s prng_t; /* opaque, library-owned */

enum {
    PRNG_OK = 0,
    PRNG_E_INVALID = -1,     /* bad argument; nothing happened */
    PRNG_E_UNSUPPORTED = -2, /* valid request outside what this build implements */
    PRNG_E_NOMEM = -3,       /* host or device allocation failed */
    PRNG_E_CUDA = -4,        /* CUDA runtime error; the handle is poisoned */
    PRNG_E_OVERRUN = -5,     /* a prng_next asked for a draw outside its epoch window */
    PRNG_E_STATE = -6        /* call not allowed in the handle's current state */
};

enum {
    PRNG_FMT_U64 = 0, /* one uint64 per number: label = x + m*y (R8) */
    PRNG_FMT_U32 = 1  /* little-endian 32-bit words of the labels (R12): one word
                         per label if m <= 2^16, else two (same bytes as U64) */
};

enum {
    PRNG_BITS_SPLITMIX = 0, /* canonical counter-addressed SplitMix64 stream (R9) */
    PRNG_BITS_RANDR = 1,    /* paper-faithful: per-walker glibc rand_r LCG streams (P:14
                               "the LCG present in the glibc library"); word k of walker t
                               = low 16 bits of outputs 2k, 2k+1 of the stream seeded with
                               low32(seed ^ (t+1)*0x9E3779B97F4A7C15) */
    PRNG_BITS_CALLBACK = 2, /* user callback supplies the words (tests, fault injection) */
    PRNG_BITS_GGCPU = 3     /* the generator itself run by the host feed threads (§IV-A
                               "Our generator, working on a multicore CPU can be used in
                               the place of rand()"; reading R23): word k of walker t = x
                               (k even) or y (k odd) of label (k mod 64)/2 of walker t of
                               the m = 2^32, l = l0 = 64 generator seeded with
                               mix64(seed ^ (k/64 + 1) * 0xD1B54A32D192ED03), whose own
                               seed bits are the SplitMix64 stream (R9).  Costs one host
                               walk of 64 steps per two words. */
};

/* Graph parameters (§III-A/B).  Paper defaults in comments. */
typedef struct {
    uint64_t m;          /* modulus: 2^32 (n = 2^65 vertices, §III-B).  Allowed:
                            any m in [2, 2^32]; powers of two take the fast
                            wrapped-arithmetic kernels, other m the generic one
                            (conditional-subtract reduction, 64-bit above 2^30) */
    uint32_t degree;     /* must be 7 (Gabber–Galil), else PRNG_E_UNSUPPORTED */
    uint32_t walk_len;   /* l = 64 steps per number (Alg.2, R6); 1..4096 */
    uint32_t burnin_len; /* l0 = 64 steps of Alg.1 ("initial walk of length 64"); 0..4096 */
    uint32_t variant;    /* 0 = forward maps sigma_k at every step (R2); 1 = bipartite
                            walk: global step s applies sigma_k (s even, X -> Y) or
                            sigma_k^{-1} (s odd, Y -> X) */
} prng_graph_params;

/*
 * Bit callback (bit_source = PRNG_BITS_CALLBACK).  Must write word
 * (word0 + r) of walker (walker0 + i) — walker ids GLOBAL — to
 * out[r * pitch + i] for r < nwords, i < nwalkers.  Word layout of one
 * walker's stream (R9): words 0,1 = start vertex; 2 .. 1+R0 = burn-in
 * record; 2+R0+R*j+r = record of draw j (R = ceil(3l/32), R0 = ceil(3l0/32)).
 * Called from library threads, possibly concurrently for disjoint ranges.
 */
typedef void (*prng_bits_fn)(void *ctx, uint64_t walker0, uint64_t nwalkers,
                             uint64_t word0, uint32_t nwords, uint32_t *out,
                             uint64_t pitch);

typedef struct {
    int device;               /* CUDA ordinal (default 0) */
    uint64_t walker_base;     /* global id of this handle's walker 0: a GPU shard owns
                                 walkers [walker_base, walker_base + walkers) */
    uint32_t epoch_draws;     /* D: draws per walker per streamed ring slot (default 16) */
    uint32_t host_threads;    /* feed threads; 0 = auto (hardware concurrency) */
    uint32_t bit_source;      /* PRNG_BITS_* */
    prng_bits_fn bits_fn;     /* for PRNG_BITS_CALLBACK */
    void *bits_ctx;
} prng_options;

/* Fill *p / *o with the paper's defaults (m = 2^32, degree 7, l = l0 = 64). */
int prng_default_params(prng_graph_params *p);
int prng_default_options(prng_options *o);

/*
 * Alg.1 InitializeGenerator (§III-B): every walker t starts at the
 * vertex given by the first 64 bits of its stream and walks l0 steps.
 * `walkers` W in [1, 2^24] (R9 counter space; W + walker_base <= 2^24).
 * Blocks until the initial walk has completed on the device.
 * `opt` may be NULL (defaults).  On success *out is a new handle.
 */
int prng_create(prng_t **out, const prng_graph_params *g, uint64_t walkers,
                uint64_t seed, const prng_options *opt);

/*
 * Bulk Alg.2 (§III-B, §IV-A): write the next n numbers of the bulk
 * sequence Z[N .. N+n) (R11: Z[g] = label of walker g mod W, draw g div W;
 * N advances by the labels written) to dev_ptr, in format fmt.
 *   dev_ptr : caller-owned device memory, >= n * (fmt==U64 ? 8 : 4) bytes,
 *             aligned to 8 bytes (labels are stored whole), or to 4 bytes
 *             for U32 with m <= 2^16 (one word per label); else
 *             PRNG_E_INVALID.
 *   n       : count in units of fmt.  For U32 with m > 2^16, n must be even.
 *   stream  : the kernels (and any copies of bits not already resident) are
 *             ordered on this stream; the call returns after enqueueing, but
 *             may block the host thread while the feed produces bits.
 * Bits of draws made resident by prng_prefetch are used directly (K-mode);
 * other draws are fed by host threads into pinned ring slots and copied on
 * a side stream, overlapped with the walk (E-mode, Fig.4 FEED/TRANSFER/
 * GENERATE).  Not allowed while an on-demand epoch is open (PRNG_E_STATE).
 * Draw indices are 32-bit: a call that would need draw 2^32 - 256 or later of
 * any walker (ceil((N + labels) / W) > 2^32 - 256) returns
 * PRNG_E_UNSUPPORTED before anything is enqueued (same for prng_prefetch,
 * prng_epoch_begin and a prng_load of such a position).
 */
int prng_fill(prng_t *h, void *dev_ptr, uint64_t n, int fmt, void *stream);

/*
 * Same as prng_fill but the numbers land in caller-owned HOST memory
 * (pinned memory strongly recommended); host<->device copies overlap the
 * walk.  Synchronous: returns when host_ptr holds all n numbers.
 */
int prng_fill_host(prng_t *h, void *host_ptr, uint64_t n, int fmt);

/*
 * Make the bits of the next `draws` draws of every walker resident in HBM
 * (FEED + TRANSFER ahead of time).  Subsequent prng_fill calls that stay
 * within those draws run the walk kernels only.  Replaces any previous
 * resident window.  Blocks until the bits are on the device.
 */
int prng_prefetch(prng_t *h, uint64_t draws);

/* Position of the bulk sequence: *n_out = N (labels generated so far). */
int prng_tell(prng_t *h, uint64_t *n_out);

/*
 * Device-side checkpoint: prng_mark saves walker state and N; prng_rewind
 * restores them (stream-ordered on `stream`), so the next fill reproduces
 * the same numbers bit-exactly (checkpoint/resume).
 */
int prng_mark(prng_t *h, void *stream);
int prng_rewind(prng_t *h, void *stream);

/*
 * Host checkpoint: prng_state_size gives the bytes of a serialised state;
 * prng_save / prng_load copy walker state + N (+ epoch cursor) to/from a
 * caller buffer of that size.  prng_load requires a handle created with the
 * same params, walkers, seed, walker_base and bit_source (the checkpoint
 * header records them; a mismatch returns PRNG_E_INVALID and changes nothing).
 */
int prng_state_size(prng_t *h, size_t *bytes);
int prng_save(prng_t *h, void *host_buf, size_t bytes);
int prng_load(prng_t *h, const void *host_buf, size_t bytes);

/* ---------------- on-demand (GetNextRand inside user kernels) ----------- */

/*
 * Open an on-demand epoch (R10): draws [J0, J0 + draws) of walkers
 * [0, active_walkers) become resident, where J0 = the epoch cursor
 * (first epoch: ceil(N / W)).  Inside the epoch a kernel may call
 * prng_next on walker t < active_walkers up to `draws` times in total (over
 * any number of launches); the i-th call returns draw J0 + i of that walker.
 * stream: the bits' H2D copy is ordered before later work on this stream.
 */
int prng_epoch_begin(prng_t *h, uint64_t active_walkers, uint32_t draws, void *stream);

/*
 * Same as prng_epoch_begin, but the window holds the walkers listed in
 * `walkers` (HOST array of `count` distinct handle-local walker indices):
 * slot k of the window (the index kernels pass to prng_state_load) is walker
 * walkers[k].  Only those walkers' bits are fed and copied; the numbers each
 * walker receives are unchanged (still draw J0 + i of that walker).
 */
int prng_epoch_begin_list(prng_t *h, const uint32_t *walkers, uint64_t count, uint32_t draws,
                          void *stream);

/* Close the epoch: cursor J0 += draws; unused draws are skipped (R10). */
int prng_epoch_end(prng_t *h, void *stream);

/*
 * Pre-allocate both device window slots (epochs are double-buffered) for
 * windows of up to `active_walkers` x `draws`, so that later
 * prng_epoch_begin calls within that size never allocate (no allocation or
 * device synchronisation jitter inside a timed or latency-sensitive loop).
 * Blocks until slots in use by earlier epochs are free.  Returns
 * PRNG_E_INVALID for zero sizes or active_walkers > walkers, PRNG_E_STATE
 * inside an open epoch.
 */
int prng_epoch_reserve(prng_t *h, uint64_t active_walkers, uint32_t draws);

/*
 * Fill *view (a struct prng_view from prng_device.cuh, view_bytes =
 * sizeof(struct prng_view)) for the open epoch.  The view holds device
 * pointers; pass it by value to kernels.
 */
int prng_device_view(prng_t *h, void *view, size_t view_bytes);

/* Read the device sticky flags: PRNG_OK, or PRNG_E_OVERRUN if any prng_next
 * ran past its window (it then returned 0).  Synchronises the device.  */
int prng_check(prng_t *h);

/* Counters for measurement (cumulative over the handle's life). */
typedef struct {
    uint64_t labels_generated;   /* bulk labels */
    uint64_t bits_bytes_fed;     /* bytes generated by the host feed */
    uint64_t h2d_bytes;          /* bytes copied host -> device */
    uint64_t d2h_bytes;          /* bytes copied device -> host */
    uint64_t kernel_launches;    /* launches of the library's kernels */
    double feed_seconds;         /* wall time host threads spent generating */
    uint32_t feed_pace_mbs;      /* SplitMix64 feed threads' aggregate streaming-store cap, MB/s:
                                    1.25 x the pinned H2D rate measured at the first create
                                    on a device (0 = unpaced; GG_FEED_RATE overrides) */
    uint32_t _reserved;
} prng_stats;
int prng_get_stats(prng_t *h, prng_stats *s);

/* Join feed threads and free everything.  NULL is a no-op (returns PRNG_OK). */
int prng_destroy(prng_t *h);

/* Static string for a status code. */
const char *prng_strerror(int status);

/* Library version, e.g. 100 for 0.1.0. */
int prng_version(void);

#ifdef __cplusplus
}
#endif
#endif /* GGPRNG_PRNG_H */

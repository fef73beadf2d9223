// Internal interfaces between the C-ABI host code and the CUDA kernels.
// Not installed; not part of the public ABI (include/prng.h is).
#pragma once
#include <cstddef>
#include <cstdint>

#include <cuda_runtime.h>

struct prng_s;

namespace gg {

// Alg.1 (§III-B) for walkers [w0, w0 + count): start vertex from stream
// words 0,1 (R7), then l0 steps with words 2 .. 1+R0.  `bits` holds rows
// 0 .. 1+R0 for those walkers, row pitch `pitch` words, walker w at column
// (w - w0).
struct InitArgs {
    const uint32_t *bits;
    uint64_t pitch;
    uint32_t w0, count;
    uint32_t l0, R0;
    uint64_t m;
    uint32_t log2m, pow2;
    uint32_t *x, *y, *j;
    uint32_t variant;
};
cudaError_t launch_init(const InitArgs &a, cudaStream_t s);

// Bulk Alg.2 over draws [ja, jb) of every walker, restricted to bulk
// positions g in [N, N + nl) (R11: g = j*W + t).  The bits of draw j are rows
// (j - Jw)*R .. (j - Jw)*R + R-1 of the window `bits` (pitch words per row).
// Writes label(g) to out[g - g_origin] (u64), or its low word (u32 when
// m <= 2^16).
struct FillArgs {
    const uint32_t *bits;
    uint64_t pitch;
    uint64_t rows;   // rows of the window (for the TMA tensor map)
    uint32_t Jw;
    uint32_t ja, jb;
    uint32_t W;
    uint64_t N, nl, g_origin;
    uint32_t *x, *y;
    void *out;
    int out_u32;
    uint32_t l, R;
    uint64_t m;
    uint32_t log2m, pow2;
    uint32_t variant, l0;
    const uint32_t *tab;  // composed-step tables (walk_table: forward, then bipartite)
};
cudaError_t launch_fill(const FillArgs &a, cudaStream_t s, int sm_count);

// Decide once per process whether the table fill kernel's shared window puts
// its table at a 16 KB boundary (ORB layout, gg_walk.cu); called by
// prng_create on a library stream (never inside a user's stream capture).
void probe_fill_layout(cudaStream_t s);

// The composed-step walk tables in global memory of the current device, built
// on first use: PRNG_TABLE_WORDS entries of the forward maps (prng_device.cuh),
// then as many of the bipartite variant's; nullptr on error.
const uint32_t *walk_table(int device);

// Host feed: SplitMix64 counter-hash stream (R9), SoA rows.
//   out[r*pitch + i] = word32(seed, tg0 + i, k0 + r),  r < nrows, i < count
// nt: stream the stores past the CPU caches (see feed.cpp).  pace_bps > 0:
// the calling thread writes at most that many bytes per second (feed.cpp Pacer).
void feed_splitmix_rows(uint64_t seed, uint64_t tg0, uint64_t count, uint64_t k0,
                        uint32_t nrows, uint32_t *out, uint64_t pitch, bool nt = false,
                        double pace_bps = 0);
// Same for an explicit walker list: column i = global walker base + ids[i].
void feed_splitmix_rows_ids(uint64_t seed, uint64_t base, const uint32_t *ids, uint64_t count,
                            uint64_t k0, uint32_t nrows, uint32_t *out, uint64_t pitch,
                            bool nt = false, double pace_bps = 0);

// Paper-faithful glibc rand_r seed bits (bit_source 1): see feed.cpp.
void feed_randr_rows(uint64_t seed, uint64_t tg0, uint64_t count, uint64_t k0, uint32_t nrows,
                     uint32_t *out, uint64_t pitch);
void feed_randr_rows_ids(uint64_t seed, uint64_t base, const uint32_t *ids, uint64_t count,
                         uint64_t k0, uint32_t nrows, uint32_t *out, uint64_t pitch);

// The generator on the host as the FEED (bit_source 3, reading R23; see
// feed.cpp).  Per walker of the handle (index = global id - t0): the host
// walk's state (x, y) after label nxt - 1 of block blk (nxt = 0: nothing
// walked yet).  Column i is global walker base + l0 + i, or base + ids[i].
struct GgCpuCache {
    uint32_t *x, *y, *blk, *nxt;
    uint64_t t0;
};
void feed_ggcpu_rows(uint64_t seed, uint64_t base, uint64_t l0, const uint32_t *ids,
                     uint64_t count, uint64_t k0, uint32_t nrows, uint32_t *out, uint64_t pitch,
                     GgCpuCache &cache);

// Stage walkers [0, hi) of the next on-demand epoch's window (one draw, row
// pitch `pitch`) ahead of prng_epoch_begin (prng_capi.cu); list ranking.
int epoch_prefeed(prng_s *h, uint64_t hi, uint64_t pitch);

// Timeline recorder of the handle (GG_TIMELINE, diagnostic; prng_capi.cu):
// host clock in us (< 0 when the recorder is off), a host interval, and a
// device interval as an event pair on stream s (tl_dev_begin returns null
// when off; tl_dev_end(h, kind, null, s) is a no-op).
double tl_now_us(prng_s *h);
void tl_host_span(prng_s *h, const char *kind, double a_us, double b_us);
cudaEvent_t tl_dev_begin(prng_s *h, cudaStream_t s);
void tl_dev_end(prng_s *h, const char *kind, cudaEvent_t a, cudaStream_t s);

// Stable single-pass compaction (compact.cu): items i < n with flags[i] != 0
// go, in order, to kept_out (the item is in[i], or i when in is null); the
// others, in order, to removed_out (if not null).  The kept count is written
// to *d_count and, if h_count (mapped pinned host memory) is given, as
// (tag << 32 | count) to *h_count once the count is final, for the host to
// poll without a device synchronisation.  scratch: compact_scratch_bytes(n)
// bytes of device memory, reset on the stream by every call.
size_t compact_scratch_bytes(int64_t n);
cudaError_t compact_flagged(const int32_t *in, const uint8_t *flags, int64_t n, int32_t *kept_out,
                            int32_t *removed_out, int32_t *d_count, volatile uint64_t *h_count,
                            uint32_t tag, void *scratch, cudaStream_t s);

// Library-owned stream-ordered scratch pool of the current device (listrank.cu):
// keeps its memory between calls; nullptr on CUDA failure.
cudaMemPool_t scratch_pool();

}  // namespace gg

// C ABI of the B200 expander-walk PRNG (declarations and contract:
// include/prng.h).  Host-side runtime: handle, feed thread pool, pinned
// staging pipeline (FEED -> TRANSFER, §IV-A Fig.4), resident and
// streamed bit windows, on-demand epochs (R10), checkpoints.
#include <algorithm>
#include <atomic>
#include <cctype>
#include <sched.h>
#include <pthread.h>
#include <chrono>
#include <condition_variable>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <functional>
#include <mutex>
#include <new>
#include <string>
#include <thread>
#include <vector>

#include <cuda_runtime.h>
#include <nvtx3/nvToolsExt.h>

#include "gg_internal.h"
#include "prng.h"
#include "prng_device.cuh"

namespace {

// ------------------------------------------------------------ thread pool
class ThreadPool {
  public:
    // cpus: if non-empty, worker i (i >= 1; index 0 is the calling thread,
    // never pinned) is pinned to cpus[i % cpus.size()].  Each worker sleeps
    // on its own condition variable, so a job for the first k threads wakes
    // only those (the SplitMix feed uses a few writers of a larger pool).
    explicit ThreadPool(unsigned n, std::vector<int> cpus = {}) : n_(n ? n : 1), slots_(n_) {
        for (unsigned i = 1; i < n_; i++)
            workers_.emplace_back([this, i, cpus] {
                if (!cpus.empty()) {
                    cpu_set_t set;
                    CPU_ZERO(&set);
                    CPU_SET(cpus[i % cpus.size()], &set);
                    pthread_setaffinity_np(pthread_self(), sizeof(set), &set);
                }
                loop(i);
            });
    }
    ~ThreadPool() {
        for (unsigned i = 1; i < n_; i++) {
            std::lock_guard<std::mutex> g(slots_[i].mu);
            slots_[i].stop = true;
            slots_[i].cv.notify_one();
        }
        for (auto &t : workers_) t.join();
    }
    unsigned size() const { return n_; }
    // fn(thread_index) on threads 0 .. k-1 (k = 0: all; the caller is thread
    // 0); returns when they are done.
    void run(const std::function<void(unsigned)> &fn, unsigned k = 0) {
        k = (k == 0 || k > n_) ? n_ : k;
        if (k == 1) {
            fn(0);
            return;
        }
        {
            std::lock_guard<std::mutex> g(done_mu_);
            pending_ = k - 1;
        }
        for (unsigned i = 1; i < k; i++) {
            std::lock_guard<std::mutex> g(slots_[i].mu);
            slots_[i].job = &fn;
            slots_[i].cv.notify_one();
        }
        fn(0);
        std::unique_lock<std::mutex> lk(done_mu_);
        done_cv_.wait(lk, [this] { return pending_ == 0; });
    }

  private:
    struct Slot {
        std::mutex mu;
        std::condition_variable cv;
        const std::function<void(unsigned)> *job = nullptr;
        bool stop = false;
    };
    void loop(unsigned idx) {
        Slot &sl = slots_[idx];
        for (;;) {
            const std::function<void(unsigned)> *job;
            {
                std::unique_lock<std::mutex> lk(sl.mu);
                sl.cv.wait(lk, [&] { return sl.stop || sl.job != nullptr; });
                if (sl.stop) return;
                job = sl.job;
                sl.job = nullptr;
            }
            (*job)(idx);
            {
                std::lock_guard<std::mutex> g(done_mu_);
                if (--pending_ == 0) done_cv_.notify_one();
            }
        }
    }
    unsigned n_;
    std::vector<Slot> slots_;
    std::vector<std::thread> workers_;
    std::mutex done_mu_;
    std::condition_variable done_cv_;
    unsigned pending_ = 0;
};

// CPUs of the GPU's own NUMA node (feed threads next to
// the GPU's PCIe root): /sys/bus/pci/devices/<bus id>/local_cpulist,
// intersected with the process's allowed CPUs; empty if unknown.
std::vector<int> gpu_local_cpus(int device) {
    std::vector<int> out;
    char bus[32] = {0};
    if (cudaDeviceGetPCIBusId(bus, sizeof(bus), device) != cudaSuccess) return out;
    for (char *c = bus; *c; c++) *c = (char)tolower(*c);
    char path[128];
    snprintf(path, sizeof(path), "/sys/bus/pci/devices/%s/local_cpulist", bus);
    FILE *f = fopen(path, "r");
    if (!f) return out;
    char line[1024] = {0};
    const bool ok = fgets(line, sizeof(line), f) != nullptr;
    fclose(f);
    if (!ok) return out;
    cpu_set_t allowed;
    CPU_ZERO(&allowed);
    if (sched_getaffinity(0, sizeof(allowed), &allowed) != 0) return out;
    for (char *tok = strtok(line, ",\n"); tok; tok = strtok(nullptr, ",\n")) {
        int a = -1, b = -1;
        if (sscanf(tok, "%d-%d", &a, &b) == 2) {
        } else if (sscanf(tok, "%d", &a) == 1) {
            b = a;
        } else {
            continue;
        }
        for (int c = a; c <= b && c < CPU_SETSIZE; c++)
            if (c >= 0 && CPU_ISSET(c, &allowed)) out.push_back(c);
    }
    return out;
}

inline uint32_t words_per_walk(uint32_t nsteps) { return (3u * nsteps + 31u) / 32u; }
inline uint64_t round_up(uint64_t v, uint64_t a) { return (v + a - 1) / a * a; }

struct CudaFail {
    cudaError_t e;
};
#define CK(call)                                    \
    do {                                            \
        cudaError_t _e = (call);                    \
        if (_e != cudaSuccess) throw CudaFail{_e};  \
    } while (0)

}  // namespace

// Fig.4 timeline (diagnostic, GG_TIMELINE=<path>): every FEED chunk (host
// interval of the feed threads), H2D copy, walk kernel and D2H copy of the
// handle as [kind, start_us, end_us] on one clock, written to <path> as JSON
// by prng_destroy.  Device intervals are event pairs on the stream the work
// ran on, placed on the host clock through a base event synchronised at
// creation (alignment error ~10 us).  Host work also carries NVTX ranges
// ("gg.feed", "gg.stage", "gg.fill") for an attached Nsight Systems.
struct Timeline {
    std::string path;
    std::chrono::steady_clock::time_point t0;
    cudaEvent_t base = nullptr;
    struct Host { const char *kind; double a, b; };
    struct Dev { const char *kind; cudaEvent_t a, b; };
    std::vector<Host> host;
    std::vector<Dev> dev;
    std::mutex mu;
    double now_us() const {
        return std::chrono::duration<double, std::micro>(std::chrono::steady_clock::now() - t0)
            .count();
    }
    void host_span(const char *kind, double a, double b) {
        std::lock_guard<std::mutex> lk(mu);
        host.push_back({kind, a, b});
    }
    // event pair around work enqueued on s between begin() and end()
    cudaEvent_t begin(cudaStream_t s) {
        cudaEvent_t e = nullptr;
        cudaEventCreate(&e);
        cudaEventRecord(e, s);
        return e;
    }
    void end(const char *kind, cudaEvent_t a, cudaStream_t s) {
        cudaEvent_t e = nullptr;
        cudaEventCreate(&e);
        cudaEventRecord(e, s);
        std::lock_guard<std::mutex> lk(mu);
        dev.push_back({kind, a, e});
    }
    void dump() {
        cudaDeviceSynchronize();
        FILE *f = fopen(path.c_str(), "w");
        if (!f) return;
        fprintf(f, "[");
        bool first = true;
        for (auto &r : host) {
            fprintf(f, "%s[\"%s\", %.3f, %.3f]", first ? "" : ",\n", r.kind, r.a, r.b);
            first = false;
        }
        for (auto &r : dev) {
            float a = 0, b = 0;
            cudaEventElapsedTime(&a, base, r.a);
            cudaEventElapsedTime(&b, base, r.b);
            fprintf(f, "%s[\"%s\", %.3f, %.3f]", first ? "" : ",\n", r.kind, a * 1e3, b * 1e3);
            first = false;
            cudaEventDestroy(r.a);
            cudaEventDestroy(r.b);
        }
        fprintf(f, "]\n");
        fclose(f);
        cudaEventDestroy(base);
    }
};

// Host FEED pace (SplitMix64 source, streaming-store windows: on-demand
// epochs < 1 GB).  A chunk is written by the pool's threads together, then
// the copy engine reads it while the next chunks are written.  Streaming
// stores from every core at once saturate host memory
// (~180 GB/s on the GPU box) and starve that DMA (55 -> 21 GB/s,
// tools/host_contention.cu, profiles/r02_host_contention.json); writers
// at ~66 GB/s leave it at 55.  So the feed threads pace themselves to an
// aggregate 1.25 x the pinned H2D rate, measured once per device per
// process (GG_FEED_RATE=<GB/s> forces a cap, 0 = unpaced).  Returns bytes/s.
double feed_rate_for(int device) {
    if (const char *e = getenv("GG_FEED_RATE")) return std::max(0.0, atof(e)) * 1e9;
    static std::mutex mu;
    static std::vector<std::pair<int, double>> cache;  // device -> bytes/s
    std::lock_guard<std::mutex> g(mu);
    for (auto &c : cache)
        if (c.first == device) return c.second;
    double h2d_gbs = 55.0;  // pinned 4 x 16 MB after one warm-up copy
    void *hp = nullptr, *dp = nullptr;
    cudaStream_t st = nullptr;
    cudaEvent_t a = nullptr, b = nullptr;
    const size_t bytes = 16u << 20;
    if (cudaHostAlloc(&hp, bytes, cudaHostAllocPortable) == cudaSuccess &&
        cudaMalloc(&dp, bytes) == cudaSuccess &&
        cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking) == cudaSuccess &&
        cudaEventCreate(&a) == cudaSuccess && cudaEventCreate(&b) == cudaSuccess) {
        memset(hp, 0, bytes);
        cudaMemcpyAsync(dp, hp, bytes, cudaMemcpyHostToDevice, st);
        cudaEventRecord(a, st);
        for (int i = 0; i < 4; i++) cudaMemcpyAsync(dp, hp, bytes, cudaMemcpyHostToDevice, st);
        cudaEventRecord(b, st);
        float ms = 0;
        if (cudaEventSynchronize(b) == cudaSuccess && cudaEventElapsedTime(&ms, a, b) == cudaSuccess &&
            ms > 0)
            h2d_gbs = 4.0 * bytes / (ms / 1e3) / 1e9;
    }
    if (a) cudaEventDestroy(a);
    if (b) cudaEventDestroy(b);
    if (st) cudaStreamDestroy(st);
    if (dp) cudaFree(dp);
    if (hp) cudaFreeHost(hp);
    cudaGetLastError();  // a failed probe keeps the default above
    const double rate = 1.25 * h2d_gbs * 1e9;
    cache.emplace_back(device, rate);
    return rate;
}

struct prng_s {
    Timeline *tl = nullptr;
    const uint32_t *walk_tab = nullptr;  // composed-step table of the device (gg::walk_table)
    prng_graph_params g{};
    prng_options o{};
    uint64_t W = 0, seed = 0;
    uint32_t R = 0, R0 = 0, log2m = 0, pow2 = 0;
    int sm_count = 148;
    bool poisoned = false;
    cudaStream_t copy_stream = nullptr;  // H2D of seed bits
    cudaStream_t d2h_stream = nullptr;   // D2H of results (prng_fill_host)
    cudaStream_t work_stream = nullptr;  // kernels of prng_fill_host
    ThreadPool *pool = nullptr;
    double feed_rate = 0;  // aggregate SplitMix feed pace, bytes/s (feed_rate_for; 0 = unpaced)

    // walker state (device) and checkpoint copies
    uint32_t *x = nullptr, *y = nullptr, *j = nullptr, *flags = nullptr;
    uint32_t *xs = nullptr, *ys = nullptr, *js = nullptr;
    uint64_t N = 0;
    uint64_t N_mark = 0, od_J0_mark = 0;
    bool have_mark = false, od_started_mark = false;

    // pinned staging chunks
    static const int kMaxChunks = 8;
    int kChunks = 4;
    uint32_t *chunk[kMaxChunks] = {};
    size_t chunk_bytes = 0;
    cudaEvent_t chunk_done[kMaxChunks] = {};
    int chunk_next = 0;

    // host walks of the generator-as-FEED bit source (PRNG_BITS_GGCPU, R23)
    std::vector<uint32_t> gg_x, gg_y, gg_blk, gg_nxt;
    uint64_t gg_t0 = 0;  // global id of cache slot 0 (the handle's walker_base)

    // resident (prefetched) window: draws [res_J, res_J + res_D) of all walkers
    uint32_t *res_bits = nullptr;
    size_t res_cap = 0;
    uint64_t res_J = 0, res_D = 0;

    // streamed ring (E-mode): 2 device slots of Ds draws
    uint32_t *ring[2] = {};
    size_t ring_cap = 0;
    cudaEvent_t ring_free[2] = {};
    int ring_next = 0;

    // prng_fill_host output staging
    void *hout[2] = {};
    size_t hout_cap = 0;
    cudaEvent_t hout_free[2] = {};

    // on-demand epoch
    bool od_open = false, od_started = false;
    uint64_t od_J0 = 0, od_Wv = 0, od_pitch = 0;
    uint32_t od_D = 0;
    uint32_t *od_bits = nullptr;       // window of the open epoch (= od_buf[od_slot])
    uint32_t *od_buf[2] = {};          // double-buffered: epoch e+1 is fed while e runs
    size_t od_cap[2] = {};
    cudaEvent_t od_free[2] = {};       // recorded at epoch_end: kernels done with the slot
    int od_slot = 1;
    // prefed part of the next epoch's window (gg_epoch_prefeed): walkers
    // [0, pf_hi) of draw pf_J0 already staged in od_buf[pf_slot] at pitch pf_pitch
    bool pf_valid = false;
    int pf_slot = 0;
    uint64_t pf_J0 = 0, pf_hi = 0, pf_pitch = 0;
    uint32_t *od_wmap_buf[2] = {};     // slot -> walker maps (prng_epoch_begin_list)
    size_t od_wmap_cap[2] = {};
    const uint32_t *od_wmap = nullptr; // map of the open epoch, or nullptr

    cudaEvent_t ev_tmp = nullptr;
    prng_stats stats{};

    uint64_t pitch() const { return round_up(W, 32); }
};

namespace {

void free_all(prng_s *h) {
    cudaSetDevice(h->o.device);
    cudaDeviceSynchronize();
    for (auto p : {h->x, h->y, h->j, h->flags, h->xs, h->ys, h->js, h->res_bits, h->ring[0],
                   h->ring[1], h->od_buf[0], h->od_buf[1], h->od_wmap_buf[0], h->od_wmap_buf[1]})
        if (p) cudaFree(p);
    for (auto p : h->hout)
        if (p) cudaFree(p);
    for (int i = 0; i < h->kChunks; i++) {
        if (h->chunk[i]) cudaFreeHost(h->chunk[i]);
        if (h->chunk_done[i]) cudaEventDestroy(h->chunk_done[i]);
    }
    for (int i = 0; i < 2; i++) {
        if (h->ring_free[i]) cudaEventDestroy(h->ring_free[i]);
        if (h->hout_free[i]) cudaEventDestroy(h->hout_free[i]);
        if (h->od_free[i]) cudaEventDestroy(h->od_free[i]);
    }
    if (h->ev_tmp) cudaEventDestroy(h->ev_tmp);
    for (auto s : {h->copy_stream, h->d2h_stream, h->work_stream})
        if (s) cudaStreamDestroy(s);
    delete h->pool;
    h->pool = nullptr;
}

// Generate rows [k0, k0+nrows) of the streams of local walkers [wa, wb)
// (or of walkers ids[wa..wb)) into buf (row pitch bpitch words), in parallel
// over walkers; streaming_stores: see feed.cpp.
void feed_chunk(prng_s *h, uint64_t wa, uint64_t wb, uint64_t k0, uint32_t nrows, uint32_t *buf,
                const uint32_t *ids, uint64_t bpitch, bool streaming_stores) {
    const uint64_t cw = wb - wa;
    const bool nt_st = streaming_stores;
    const unsigned nt = h->pool->size();
    // streaming stores are paced (feed_rate_for); cached stores (long bulk
    // streams) are not: they measured faster unpaced (C2 E-mode 2.04 vs 1.74
    // G/s streaming unpaced, 1.90 streaming paced, tools/feed_ab.py)
    const double pace = nt_st ? h->feed_rate / nt : 0.0;  // bytes/s per thread
    auto t0 = std::chrono::steady_clock::now();
    const double tl0 = h->tl ? h->tl->now_us() : 0.0;
    nvtxRangePushA("gg.feed");
    static const bool static_slices = getenv("GG_FEED_STATIC") != nullptr;  // A/B hook
    if (h->o.bit_source == PRNG_BITS_SPLITMIX && !static_slices) {
        // Blocks of kBlk walkers claimed in order from a shared counter; on
        // streaming-store (paced) windows block b is released at t0 + (bytes
        // before b) / feed_rate.  One clock for the whole pool: a worker that
        // wakes late or is descheduled leaves its blocks to the others
        // instead of finishing the chunk late (per-thread slices with
        // per-thread pacing made each chunk as slow as its slowest writer:
        // C3 67.3 -> 66.4 ms; cached-store bulk streams: C2 e2e 2.00-2.03 ->
        // 2.02-2.08 G/s, feed time per step 0.17 -> 0.15 s).
        constexpr uint64_t kBlk = 4096;  // 16 KB per row, 64 B aligned
        const uint64_t nblk = (cw + kBlk - 1) / kBlk;
        const double blk_s =
            nt_st && h->feed_rate > 0 ? (double)kBlk * nrows * 4 / h->feed_rate : 0.0;
        std::atomic<uint64_t> next{0};
        h->pool->run([&](unsigned) {
            for (;;) {
                const uint64_t b = next.fetch_add(1, std::memory_order_relaxed);
                if (b >= nblk) return;
                if (blk_s > 0) {
                    const double due = (double)b * blk_s;
                    while (std::chrono::duration<double>(std::chrono::steady_clock::now() - t0)
                               .count() < due) {
#if defined(__x86_64__)
                        __builtin_ia32_pause();
#endif
                    }
                }
                const uint64_t lo = b * kBlk, hi = std::min(cw, lo + kBlk);
                if (ids)
                    gg::feed_splitmix_rows_ids(h->seed, h->o.walker_base, ids + wa + lo, hi - lo,
                                               k0, nrows, buf + lo, bpitch, nt_st, 0.0);
                else
                    gg::feed_splitmix_rows(h->seed, h->o.walker_base + wa + lo, hi - lo, k0, nrows,
                                           buf + lo, bpitch, nt_st, 0.0);
            }
        });
    } else {
    h->pool->run([&](unsigned ti) {
        // contiguous, 16-walker aligned slices
        uint64_t per = round_up((cw + nt - 1) / nt, 16);
        uint64_t lo = std::min<uint64_t>(cw, per * ti), hi = std::min<uint64_t>(cw, lo + per);
        if (lo >= hi) return;
        if (h->o.bit_source == PRNG_BITS_GGCPU) {
            gg::GgCpuCache c{h->gg_x.data(), h->gg_y.data(), h->gg_blk.data(), h->gg_nxt.data(),
                             h->gg_t0};
            gg::feed_ggcpu_rows(h->seed, h->o.walker_base, wa + lo, ids ? ids + wa + lo : nullptr,
                                hi - lo, k0, nrows, buf + lo, bpitch, c);
            return;
        }
        if (ids) {
            if (h->o.bit_source == PRNG_BITS_RANDR) {
                gg::feed_randr_rows_ids(h->seed, h->o.walker_base, ids + wa + lo, hi - lo, k0,
                                        nrows, buf + lo, bpitch);
            } else if (h->o.bit_source == PRNG_BITS_CALLBACK) {
                for (uint64_t i = lo; i < hi; i++)  // one walker at a time
                    h->o.bits_fn(h->o.bits_ctx, h->o.walker_base + ids[wa + i], 1, k0, nrows,
                                 buf + i, bpitch);
            } else {
                gg::feed_splitmix_rows_ids(h->seed, h->o.walker_base, ids + wa + lo, hi - lo, k0,
                                           nrows, buf + lo, bpitch, nt_st, pace);
            }
            return;
        }
        const uint64_t tg0 = h->o.walker_base + wa + lo;
        if (h->o.bit_source == PRNG_BITS_RANDR)
            gg::feed_randr_rows(h->seed, tg0, hi - lo, k0, nrows, buf + lo, bpitch);
        else if (h->o.bit_source == PRNG_BITS_CALLBACK)
            h->o.bits_fn(h->o.bits_ctx, tg0, hi - lo, k0, nrows, buf + lo, bpitch);
        else
            gg::feed_splitmix_rows(h->seed, tg0, hi - lo, k0, nrows, buf + lo, bpitch, nt_st, pace);
    });
    }
    nvtxRangePop();
    if (h->tl) h->tl->host_span("feed", tl0, h->tl->now_us());
    auto t1 = std::chrono::steady_clock::now();
    h->stats.feed_seconds += std::chrono::duration<double>(t1 - t0).count();
    h->stats.bits_bytes_fed += (uint64_t)nrows * cw * 4;
}

// H2D copy of a fed chunk on the copy stream (timeline: one "h2d" span).
void h2d_copy(prng_s *h, void *dst, const void *src, size_t bytes) {
    cudaEvent_t a = h->tl ? h->tl->begin(h->copy_stream) : nullptr;
    CK(cudaMemcpyAsync(dst, src, bytes, cudaMemcpyHostToDevice, h->copy_stream));
    if (a) h->tl->end("h2d", a, h->copy_stream);
}

// FEED + TRANSFER: stream words [k0, k0+nrows) of local walkers [0, Wv) into
// the device window dst (row pitch dpitch words).  Host threads generate a
// pinned chunk while the previous chunks are DMA'd on copy_stream.
// On return every copy is enqueued on copy_stream.
void stage_rows(prng_s *h, uint64_t k0, uint64_t nrows, uint64_t Wv, uint32_t *dst,
                uint64_t dpitch, const uint32_t *ids = nullptr, bool bursty = false,
                bool row_segments = false) {
    if (nrows == 0 || Wv == 0) return;
    static const bool nt_all = getenv("GG_FEED_NT_ALL") != nullptr;  // A/B hook
    bursty = bursty || nt_all;
    const uint64_t chunk_words = h->chunk_bytes / 4;
    // Chunks hold an even number of rows (>= 2) so each 64-bit SplitMix word
    // feeds two rows (k even, k+1) with one hash.  Full-width chunks are
    // generated at the device pitch, so each is ONE contiguous DMA (a 2D copy
    // with pitch != width ran at 14-26 GB/s instead of ~46); windows wider
    // than half a chunk are split by walkers, one contiguous DMA per row.
    static const bool trace = getenv("GG_FEED_TRACE") != nullptr;
    cudaEvent_t tr0 = nullptr, tr1 = nullptr;
    auto host_t0 = std::chrono::steady_clock::now();
    if (trace) {
        cudaEventCreate(&tr0);
        cudaEventCreate(&tr1);
        cudaEventRecord(tr0, h->copy_stream);
    }
    struct TraceEnd {
        prng_s *h;
        cudaEvent_t a, b;
        std::chrono::steady_clock::time_point t0;
        uint64_t bytes0;
        ~TraceEnd() {
            if (!a) return;
            cudaEventRecord(b, h->copy_stream);
            auto t1 = std::chrono::steady_clock::now();
            cudaEventSynchronize(b);
            auto t2 = std::chrono::steady_clock::now();
            float ms = 0;
            cudaEventElapsedTime(&ms, a, b);
            fprintf(stderr, "[feed] %.1f MB: host gen+enqueue %.3f ms, copy stream %.3f ms (events), "
                    "host wait after enqueue %.3f ms\n",
                    (h->stats.h2d_bytes - bytes0) / 1e6,
                    std::chrono::duration<double, std::milli>(t1 - t0).count(), ms,
                    std::chrono::duration<double, std::milli>(t2 - t1).count());
            cudaEventDestroy(a);
            cudaEventDestroy(b);
        }
    } trace_end{h, tr0, tr1, host_t0, h->stats.h2d_bytes};
    // row_segments: copy only columns [0, Wv) of every row (dst may point into
    // the middle of a row); otherwise small windows go as whole-row chunks
    if (2 * dpitch <= chunk_words && !row_segments) {
        uint64_t rows_per = std::max<uint64_t>(2, (chunk_words / dpitch) & ~1ull);
        for (uint64_t r = 0; r < nrows;) {
            uint64_t nr = std::min<uint64_t>(rows_per, nrows - r);
            if (((k0 + r) & 1) && nr > 1) nr -= 1;  // keep later chunks pair-aligned
            const int b = h->chunk_next;
            h->chunk_next = (b + 1) % h->kChunks;
            {  // pinned chunk free again
                const double w0 = h->tl ? h->tl->now_us() : 0.0;
                CK(cudaEventSynchronize(h->chunk_done[b]));
                if (h->tl) h->tl->host_span("ring_wait", w0, h->tl->now_us());
            }
            feed_chunk(h, 0, Wv, k0 + r, (uint32_t)nr, h->chunk[b], ids, dpitch, bursty);
            h2d_copy(h, dst + r * dpitch, h->chunk[b], nr * dpitch * 4);
            CK(cudaEventRecord(h->chunk_done[b], h->copy_stream));
            h->stats.h2d_bytes += nr * dpitch * 4;
            r += nr;
        }
        return;
    }
    const uint64_t walkers_per = std::max<uint64_t>(32, (chunk_words / 2) & ~31ull);
    for (uint64_t r = 0; r < nrows;) {
        uint64_t nr = std::min<uint64_t>(2, nrows - r);
        if (((k0 + r) & 1) && nr > 1) nr = 1;
        for (uint64_t wa = 0; wa < Wv; wa += walkers_per) {
            const uint64_t wb = std::min<uint64_t>(Wv, wa + walkers_per);
            const int b = h->chunk_next;
            h->chunk_next = (b + 1) % h->kChunks;
            {
                const double w0 = h->tl ? h->tl->now_us() : 0.0;
                CK(cudaEventSynchronize(h->chunk_done[b]));
                if (h->tl) h->tl->host_span("ring_wait", w0, h->tl->now_us());
            }
            const uint64_t cw = wb - wa;
            // rows start 32-B aligned in the chunk, so the streaming-store path
            // (feed.cpp nt_ok) covers the ragged last segment too: cached
            // stores there halved the DMA rate of whole rounds (LR trace)
            const uint64_t cp = round_up(cw, 8);
            feed_chunk(h, wa, wb, k0 + r, (uint32_t)nr, h->chunk[b], ids, cp, bursty);
            for (uint64_t i = 0; i < nr; i++)  // one contiguous DMA per row segment
                h2d_copy(h, dst + (r + i) * dpitch + wa, h->chunk[b] + i * cp, cw * 4);
            CK(cudaEventRecord(h->chunk_done[b], h->copy_stream));
            h->stats.h2d_bytes += (uint64_t)nr * cw * 4;
        }
        r += nr;
    }
}

// Make `s` wait for everything enqueued so far on copy_stream.
void join_copies(prng_s *h, cudaStream_t s) {
    CK(cudaEventRecord(h->ev_tmp, h->copy_stream));
    CK(cudaStreamWaitEvent(s, h->ev_tmp, 0));
}

void ensure_dev(uint32_t *&p, size_t &cap, size_t bytes) {
    if (bytes <= cap && p) return;
    if (p) CK(cudaFree(p));
    p = nullptr;
    cap = 0;
    CK(cudaMalloc(&p, bytes));
    cap = bytes;
}

uint64_t labels_of(const prng_s *h, uint64_t n, int fmt) {
    if (fmt == PRNG_FMT_U64) return n;
    return (h->g.m <= 65536ull) ? n : n / 2;
}

int check_fmt(const prng_s *h, uint64_t n, int fmt) {
    if (fmt != PRNG_FMT_U64 && fmt != PRNG_FMT_U32) return PRNG_E_INVALID;
    if (fmt == PRNG_FMT_U32 && h->g.m > 65536ull && (n & 1)) return PRNG_E_INVALID;
    return PRNG_OK;
}

// Draw indices are 32-bit in the walk kernels (FillArgs::Jw/ja/jb, the
// per-walker cursor j[]), and the kernels' loops step them by up to 2 draws
// and look up to 16 draws ahead: a bulk call whose end ceil((N + nl) / W)
// exceeds kDrawLimit = 2^32 - 256 is refused up front (PRNG_E_UNSUPPORTED,
// nothing enqueued), so no loop index can wrap.
constexpr uint64_t kDrawLimit = 0xFFFFFF00ull;
bool draws_fit(const prng_s *h, uint64_t N, uint64_t nl) {
    const uint64_t W = h->W;
    if (nl > UINT64_MAX - N - W) return false;
    return (N + nl + W - 1) / W <= kDrawLimit;
}

gg::FillArgs fill_args(prng_s *h, const uint32_t *bits, uint64_t pitch, uint64_t rows,
                       uint64_t Jw, uint64_t ja, uint64_t jb, uint64_t N, uint64_t nl,
                       uint64_t g_origin, void *out, int out_u32) {
    gg::FillArgs a{};
    a.bits = bits;
    a.pitch = pitch;
    a.rows = rows;
    a.Jw = (uint32_t)Jw;
    a.ja = (uint32_t)ja;
    a.jb = (uint32_t)jb;
    a.W = (uint32_t)h->W;
    a.N = N;
    a.nl = nl;
    a.g_origin = g_origin;
    a.x = h->x;
    a.y = h->y;
    a.out = out;
    a.out_u32 = out_u32;
    a.l = h->g.walk_len;
    a.R = h->R;
    a.m = h->g.m;
    a.log2m = h->log2m;
    a.pow2 = h->pow2;
    a.variant = h->g.variant;
    a.l0 = h->g.burnin_len;
    a.tab = h->walk_tab;
    return a;
}

// Core of prng_fill / prng_fill_host: draws [jlo, jhi) covering labels
// [N, N+nl).  emit(ja, jb, bits, pitch, Jw) launches the walk for one piece.
template <class Emit>
void run_pieces(prng_s *h, uint64_t N, uint64_t nl, cudaStream_t s, Emit emit) {
    const uint64_t W = h->W;
    const uint64_t jlo = N / W, jhi = (N + nl + W - 1) / W;
    const uint64_t Ds = std::max<uint32_t>(1, h->o.epoch_draws);
    const uint64_t pitch = h->pitch();
    uint64_t j = jlo;
    while (j < jhi) {
        if (h->res_bits && j >= h->res_J && j < h->res_J + h->res_D) {
            const uint64_t jb = std::min(jhi, h->res_J + h->res_D);
            emit(j, jb, h->res_bits, pitch, h->res_D * h->R, h->res_J, s);
            j = jb;
            continue;
        }
        uint64_t jb = std::min(jhi, j + Ds);
        if (h->res_bits && h->res_J > j && h->res_J < jb) jb = h->res_J;
        const int slot = h->ring_next;
        h->ring_next ^= 1;
        const size_t rbytes = (size_t)Ds * h->R * pitch * 4;
        if (h->ring_cap < rbytes) {
            CK(cudaDeviceSynchronize());
            for (auto &p : h->ring) {
                if (p) CK(cudaFree(p));
                p = nullptr;
            }
            h->ring_cap = 0;
            for (auto &p : h->ring) CK(cudaMalloc(&p, rbytes));
            h->ring_cap = rbytes;
        }
        CK(cudaStreamWaitEvent(h->copy_stream, h->ring_free[slot], 0));  // slot no longer read
        stage_rows(h, 2 + h->R0 + h->R * j, (jb - j) * h->R, W, h->ring[slot], pitch);
        join_copies(h, s);
        emit(j, jb, h->ring[slot], pitch, (jb - j) * h->R, j, s);
        CK(cudaEventRecord(h->ring_free[slot], s));
        j = jb;
    }
}

int guard(prng_s *h, const std::function<int()> &fn) {
    if (!h) return PRNG_E_INVALID;
    if (h->poisoned) return PRNG_E_STATE;
    try {
        CK(cudaSetDevice(h->o.device));
        return fn();
    } catch (const CudaFail &f) {
        fprintf(stderr, "[ggprng] CUDA error: %s\n", cudaGetErrorString(f.e));
        h->poisoned = true;
        return PRNG_E_CUDA;
    } catch (const std::bad_alloc &) {
        return PRNG_E_NOMEM;
    }
}

}  // namespace

extern "C" {

int prng_version(void) { return 100; }

const char *prng_strerror(int status) {
    switch (status) {
        case PRNG_OK: return "ok";
        case PRNG_E_INVALID: return "invalid argument";
        case PRNG_E_UNSUPPORTED: return "unsupported parameters";
        case PRNG_E_NOMEM: return "out of memory";
        case PRNG_E_CUDA: return "CUDA error (handle poisoned)";
        case PRNG_E_OVERRUN: return "on-demand draw outside the epoch window";
        case PRNG_E_STATE: return "call not allowed in the current state";
        default: return "unknown status";
    }
}

int prng_default_params(prng_graph_params *p) {
    if (!p) return PRNG_E_INVALID;
    p->m = 1ull << 32;
    p->degree = 7;
    p->walk_len = 64;
    p->burnin_len = 64;
    p->variant = 0;
    return PRNG_OK;
}

int prng_default_options(prng_options *o) {
    if (!o) return PRNG_E_INVALID;
    memset(o, 0, sizeof(*o));
    o->device = 0;
    o->walker_base = 0;
    o->epoch_draws = 16;
    o->host_threads = 0;
    o->bit_source = PRNG_BITS_SPLITMIX;
    return PRNG_OK;
}

int prng_create(prng_t **out, const prng_graph_params *g, uint64_t walkers, uint64_t seed,
                const prng_options *opt) {
    if (!out || !g) return PRNG_E_INVALID;
    *out = nullptr;
    if (walkers == 0) return PRNG_E_INVALID;
    prng_options o;
    if (opt)
        o = *opt;
    else
        prng_default_options(&o);
    if (g->degree != 7 || g->variant > 1) return PRNG_E_UNSUPPORTED;
    if (g->m < 2 || g->m > (1ull << 32)) return PRNG_E_INVALID;
    const bool pow2 = (g->m & (g->m - 1)) == 0;
    if (g->walk_len < 1 || g->walk_len > 4096 || g->burnin_len > 4096) return PRNG_E_INVALID;
    if (walkers + o.walker_base > (1ull << 24)) return PRNG_E_INVALID;
    if (o.bit_source != PRNG_BITS_SPLITMIX && o.bit_source != PRNG_BITS_RANDR &&
        o.bit_source != PRNG_BITS_CALLBACK && o.bit_source != PRNG_BITS_GGCPU)
        return PRNG_E_INVALID;
    if (o.bit_source == PRNG_BITS_CALLBACK && !o.bits_fn) return PRNG_E_INVALID;
    if (o.epoch_draws == 0) o.epoch_draws = 16;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || o.device < 0 || o.device >= ndev)
        return PRNG_E_INVALID;

    prng_s *h = new (std::nothrow) prng_s();
    if (!h) return PRNG_E_NOMEM;
    h->g = *g;
    h->o = o;
    h->W = walkers;
    h->seed = seed;
    if (o.bit_source == PRNG_BITS_GGCPU) {
        try {
            for (auto *v : {&h->gg_x, &h->gg_y, &h->gg_blk, &h->gg_nxt}) v->assign(walkers, 0u);
            h->gg_t0 = o.walker_base;
        } catch (const std::bad_alloc &) {
            delete h;
            return PRNG_E_NOMEM;
        }
    }
    h->R = words_per_walk(g->walk_len);
    h->R0 = words_per_walk(g->burnin_len);
    h->pow2 = pow2 ? 1 : 0;
    h->log2m = 0;
    if (pow2)
        while ((1ull << h->log2m) < g->m) h->log2m++;
    try {
        CK(cudaSetDevice(o.device));
        CK(cudaDeviceGetAttribute(&h->sm_count, cudaDevAttrMultiProcessorCount, o.device));
        unsigned nt = o.host_threads ? o.host_threads : std::thread::hardware_concurrency();
        if (nt == 0) nt = 1;
        // A/B hook GG_FEED_PIN=1: pin the feed threads to the GPU's NUMA-local
        // CPUs, rank r of a node (walker_base = r * walkers) on its own slice
        static const bool pin = getenv("GG_FEED_PIN") && atoi(getenv("GG_FEED_PIN")) == 1;
        std::vector<int> cpus;
        if (pin) {
            std::vector<int> local = gpu_local_cpus(o.device);
            if (!local.empty()) {
                const size_t rank = (size_t)(o.walker_base / walkers);
                for (unsigned i = 0; i < nt; i++)
                    cpus.push_back(local[(rank * nt + i) % local.size()]);
            }
        }
        h->pool = new ThreadPool(nt, cpus);
        h->feed_rate = h->o.bit_source == PRNG_BITS_SPLITMIX ? feed_rate_for(o.device) : 0.0;
        h->stats.feed_pace_mbs = (uint32_t)(h->feed_rate / 1e6);
        h->walk_tab = gg::walk_table(o.device);
        if (!h->walk_tab) CK(cudaErrorMemoryAllocation);
        if (const char *tp = getenv("GG_TIMELINE")) {
            h->tl = new Timeline();
            h->tl->path = tp;
            CK(cudaEventCreate(&h->tl->base));
            CK(cudaEventRecord(h->tl->base, nullptr));
            CK(cudaEventSynchronize(h->tl->base));
            h->tl->t0 = std::chrono::steady_clock::now();
        }
        CK(cudaStreamCreateWithFlags(&h->copy_stream, cudaStreamNonBlocking));
        CK(cudaStreamCreateWithFlags(&h->d2h_stream, cudaStreamNonBlocking));
        CK(cudaStreamCreateWithFlags(&h->work_stream, cudaStreamNonBlocking));
        gg::probe_fill_layout(h->work_stream);
        CK(cudaEventCreateWithFlags(&h->ev_tmp, cudaEventDisableTiming));
        static const int chunk_mb = getenv("GG_FEED_CHUNK_MB") ? atoi(getenv("GG_FEED_CHUNK_MB")) : 16;
        static const int nchunks = getenv("GG_FEED_CHUNKS") ? atoi(getenv("GG_FEED_CHUNKS")) : 4;
        h->chunk_bytes = (size_t)(chunk_mb > 0 ? chunk_mb : 32) << 20;
        h->kChunks = std::min(prng_s::kMaxChunks, std::max(2, nchunks));
        for (int i = 0; i < h->kChunks; i++) {
            CK(cudaHostAlloc((void **)&h->chunk[i], h->chunk_bytes, cudaHostAllocPortable));
            CK(cudaEventCreateWithFlags(&h->chunk_done[i], cudaEventDisableTiming));
        }
        for (int i = 0; i < 2; i++) {
            CK(cudaEventCreateWithFlags(&h->ring_free[i], cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&h->hout_free[i], cudaEventDisableTiming));
            CK(cudaEventCreateWithFlags(&h->od_free[i], cudaEventDisableTiming));
        }
        const size_t sb = (size_t)walkers * 4;
        for (uint32_t **p : {&h->x, &h->y, &h->j, &h->xs, &h->ys, &h->js}) CK(cudaMalloc(p, sb));
        CK(cudaMalloc(&h->flags, 4));
        CK(cudaMemset(h->flags, 0, 4));
        // Alg.1, in walker chunks to bound the temporary window.
        const uint64_t chunkW = std::min<uint64_t>(walkers, 1ull << 22);
        const uint64_t cpitch = round_up(chunkW, 32);
        uint32_t *tmp = nullptr;
        size_t tmp_cap = 0;
        ensure_dev(tmp, tmp_cap, (size_t)(2 + h->R0) * cpitch * 4);
        for (uint64_t w0 = 0; w0 < walkers; w0 += chunkW) {
            const uint64_t cnt = std::min<uint64_t>(chunkW, walkers - w0);
            // stage_rows works on walkers [0, Wv) of the handle; shift the base.
            const uint64_t saved_base = h->o.walker_base;
            h->o.walker_base = saved_base + w0;
            // one burst per chunk (<= 134 MB): streaming stores, like the on-demand
            // windows (cached stores left dirty lines that slowed the DMA to 17 GB/s)
            stage_rows(h, 0, 2 + h->R0, cnt, tmp, cpitch, nullptr, true);
            h->o.walker_base = saved_base;
            join_copies(h, h->work_stream);
            gg::InitArgs a{};
            a.bits = tmp;
            a.pitch = cpitch;
            a.w0 = (uint32_t)w0;
            a.count = (uint32_t)cnt;
            a.l0 = g->burnin_len;
            a.R0 = h->R0;
            a.m = g->m;
            a.log2m = h->log2m;
            a.pow2 = h->pow2;
            a.variant = g->variant;
            a.x = h->x;
            a.y = h->y;
            a.j = h->j;
            CK(gg::launch_init(a, h->work_stream));
            h->stats.kernel_launches++;
            CK(cudaStreamSynchronize(h->work_stream));
        }
        CK(cudaFree(tmp));
        CK(cudaDeviceSynchronize());
    } catch (const CudaFail &f) {
        fprintf(stderr, "[ggprng] CUDA error in prng_create: %s\n", cudaGetErrorString(f.e));
        free_all(h);
        delete h;
        return (f.e == cudaErrorMemoryAllocation) ? PRNG_E_NOMEM : PRNG_E_CUDA;
    } catch (const std::bad_alloc &) {
        free_all(h);
        delete h;
        return PRNG_E_NOMEM;
    }
    *out = h;
    return PRNG_OK;
}

int prng_fill(prng_t *h, void *dev_ptr, uint64_t n, int fmt, void *stream) {
    if (!h) return PRNG_E_INVALID;
    int rc = check_fmt(h, n, fmt);
    if (rc != PRNG_OK) return rc;
    if (n == 0) return PRNG_OK;
    // labels are stored whole: 8-byte alignment unless one u32 word per label
    const uintptr_t align = (fmt == PRNG_FMT_U32 && h->g.m <= 65536ull) ? 4 : 8;
    if (!dev_ptr || ((uintptr_t)dev_ptr % align)) return PRNG_E_INVALID;
    if (h->od_open) return PRNG_E_STATE;
    if (!draws_fit(h, h->N, labels_of(h, n, fmt))) return PRNG_E_UNSUPPORTED;
    return guard(h, [&] {
        cudaStream_t s = (cudaStream_t)stream;
        const uint64_t nl = labels_of(h, n, fmt);
        const int out_u32 = (fmt == PRNG_FMT_U32 && h->g.m <= 65536ull) ? 1 : 0;
        const uint64_t N = h->N;
        run_pieces(h, N, nl, s,
                   [&](uint64_t ja, uint64_t jb, const uint32_t *bits, uint64_t pitch,
                       uint64_t rows, uint64_t Jw, cudaStream_t st) {
                       gg::FillArgs a = fill_args(h, bits, pitch, rows, Jw, ja, jb, N, nl, N,
                                                  dev_ptr, out_u32);
                       cudaEvent_t ta = h->tl ? h->tl->begin(st) : nullptr;
                       CK(gg::launch_fill(a, st, h->sm_count));
                       if (ta) h->tl->end("walk", ta, st);
                       h->stats.kernel_launches++;
                   });
        h->N = N + nl;
        h->od_started = false;  // the next epoch starts at the next whole draw after N (R10)
        h->stats.labels_generated += nl;
        return PRNG_OK;
    });
}

int prng_fill_host(prng_t *h, void *host_ptr, uint64_t n, int fmt) {
    if (!h) return PRNG_E_INVALID;
    int rc = check_fmt(h, n, fmt);
    if (rc != PRNG_OK) return rc;
    if (n == 0) return PRNG_OK;
    if (!host_ptr) return PRNG_E_INVALID;
    if (h->od_open) return PRNG_E_STATE;
    if (!draws_fit(h, h->N, labels_of(h, n, fmt))) return PRNG_E_UNSUPPORTED;
    return guard(h, [&] {
        const uint64_t nl = labels_of(h, n, fmt);
        const int out_u32 = (fmt == PRNG_FMT_U32 && h->g.m <= 65536ull) ? 1 : 0;
        const size_t esz = out_u32 ? 4 : 8;
        const uint64_t N = h->N;
        const uint64_t Ds = std::max<uint32_t>(1, h->o.epoch_draws);
        const size_t need = (size_t)(Ds + 1) * h->W * esz;
        if (h->hout_cap < need) {
            for (auto &p : h->hout)
                if (p) {
                    CK(cudaFree(p));
                    p = nullptr;
                }
            for (auto &p : h->hout) CK(cudaMalloc(&p, need));
            h->hout_cap = need;
        }
        int oslot = 0;
        char *dst = (char *)host_ptr;
        cudaStream_t s = h->work_stream;
        run_pieces(h, N, nl, s,
                   [&](uint64_t ja, uint64_t jb, const uint32_t *bits, uint64_t pitch,
                       uint64_t rows, uint64_t Jw, cudaStream_t st) {
                       // a resident window may span many ring slots' worth: split
                       for (uint64_t a0 = ja; a0 < jb; a0 += Ds) {
                           const uint64_t a1 = std::min(jb, a0 + Ds);
                           const uint64_t gA = std::max(N, a0 * h->W);
                           const uint64_t gB = std::min(N + nl, a1 * h->W);
                           if (gB <= gA) continue;
                           CK(cudaStreamWaitEvent(st, h->hout_free[oslot], 0));
                           gg::FillArgs a = fill_args(h, bits, pitch, rows, Jw, a0, a1, N, nl,
                                                      gA, h->hout[oslot], out_u32);
                           cudaEvent_t ta = h->tl ? h->tl->begin(st) : nullptr;
                           CK(gg::launch_fill(a, st, h->sm_count));
                           if (ta) h->tl->end("walk", ta, st);
                           h->stats.kernel_launches++;
                           CK(cudaEventRecord(h->ev_tmp, st));
                           CK(cudaStreamWaitEvent(h->d2h_stream, h->ev_tmp, 0));
                           cudaEvent_t tc = h->tl ? h->tl->begin(h->d2h_stream) : nullptr;
                           CK(cudaMemcpyAsync(dst + (gA - N) * esz, h->hout[oslot],
                                              (gB - gA) * esz, cudaMemcpyDeviceToHost,
                                              h->d2h_stream));
                           if (tc) h->tl->end("d2h", tc, h->d2h_stream);
                           CK(cudaEventRecord(h->hout_free[oslot], h->d2h_stream));
                           h->stats.d2h_bytes += (gB - gA) * esz;
                           oslot ^= 1;
                       }
                   });
        CK(cudaStreamSynchronize(h->d2h_stream));
        CK(cudaStreamSynchronize(s));
        h->N = N + nl;
        h->od_started = false;  // the next epoch starts at the next whole draw after N (R10)
        h->stats.labels_generated += nl;
        return PRNG_OK;
    });
}

int prng_prefetch(prng_t *h, uint64_t draws) {
    if (!h) return PRNG_E_INVALID;
    if (draws == 0) return PRNG_E_INVALID;
    if (h->od_open) return PRNG_E_STATE;
    if (h->N / h->W + draws > kDrawLimit) return PRNG_E_UNSUPPORTED;
    return guard(h, [&] {
        const uint64_t pitch = h->pitch();
        const size_t bytes = (size_t)draws * h->R * pitch * 4;
        CK(cudaDeviceSynchronize());  // the old window may still be read
        ensure_dev(h->res_bits, h->res_cap, bytes);
        const uint64_t J = h->N / h->W;
        stage_rows(h, 2 + h->R0 + h->R * J, draws * h->R, h->W, h->res_bits, pitch);
        CK(cudaStreamSynchronize(h->copy_stream));
        h->res_J = J;
        h->res_D = draws;
        return PRNG_OK;
    });
}

int prng_tell(prng_t *h, uint64_t *n_out) {
    if (!h || !n_out) return PRNG_E_INVALID;
    *n_out = h->N;
    return PRNG_OK;
}

int prng_mark(prng_t *h, void *stream) {
    if (!h) return PRNG_E_INVALID;
    return guard(h, [&] {
        cudaStream_t s = (cudaStream_t)stream;
        const size_t sb = h->W * 4;
        CK(cudaMemcpyAsync(h->xs, h->x, sb, cudaMemcpyDeviceToDevice, s));
        CK(cudaMemcpyAsync(h->ys, h->y, sb, cudaMemcpyDeviceToDevice, s));
        CK(cudaMemcpyAsync(h->js, h->j, sb, cudaMemcpyDeviceToDevice, s));
        h->N_mark = h->N;
        h->od_J0_mark = h->od_J0;
        h->od_started_mark = h->od_started;
        h->have_mark = true;
        return PRNG_OK;
    });
}

int prng_rewind(prng_t *h, void *stream) {
    if (!h) return PRNG_E_INVALID;
    if (!h->have_mark || h->od_open) return PRNG_E_STATE;
    return guard(h, [&] {
        cudaStream_t s = (cudaStream_t)stream;
        const size_t sb = h->W * 4;
        CK(cudaMemcpyAsync(h->x, h->xs, sb, cudaMemcpyDeviceToDevice, s));
        CK(cudaMemcpyAsync(h->y, h->ys, sb, cudaMemcpyDeviceToDevice, s));
        CK(cudaMemcpyAsync(h->j, h->js, sb, cudaMemcpyDeviceToDevice, s));
        h->N = h->N_mark;
        h->od_J0 = h->od_J0_mark;
        h->od_started = h->od_started_mark;
        return PRNG_OK;
    });
}

namespace {
// Everything that selects the walkers' bit streams and walk is part of the
// header, so a checkpoint loads only into a handle that would have produced
// it (another shard's walker_base, variant, burn-in or bit source is refused).
struct SavedHeader {
    uint64_t magic, W, N, od_J0, od_started, m, seed, walk_len;
    uint64_t burnin_len, variant, walker_base, bit_source;
};
const uint64_t kMagic = 0x47475052'4e470002ull;
}  // namespace

int prng_state_size(prng_t *h, size_t *bytes) {
    if (!h || !bytes) return PRNG_E_INVALID;
    *bytes = sizeof(SavedHeader) + 3 * h->W * 4;
    return PRNG_OK;
}

int prng_save(prng_t *h, void *host_buf, size_t bytes) {
    if (!h || !host_buf || bytes < sizeof(SavedHeader) + 3 * h->W * 4) return PRNG_E_INVALID;
    if (h->od_open) return PRNG_E_STATE;
    return guard(h, [&] {
        SavedHeader hd{kMagic,           h->W,           h->N,
                       h->od_J0,         h->od_started ? 1ull : 0ull,
                       h->g.m,           h->seed,        h->g.walk_len,
                       h->g.burnin_len,  h->g.variant,   h->o.walker_base,
                       h->o.bit_source};
        CK(cudaDeviceSynchronize());
        memcpy(host_buf, &hd, sizeof(hd));
        char *p = (char *)host_buf + sizeof(hd);
        CK(cudaMemcpy(p, h->x, h->W * 4, cudaMemcpyDeviceToHost));
        CK(cudaMemcpy(p + h->W * 4, h->y, h->W * 4, cudaMemcpyDeviceToHost));
        CK(cudaMemcpy(p + 2 * h->W * 4, h->j, h->W * 4, cudaMemcpyDeviceToHost));
        return PRNG_OK;
    });
}

int prng_load(prng_t *h, const void *host_buf, size_t bytes) {
    if (!h || !host_buf || bytes < sizeof(SavedHeader) + 3 * h->W * 4) return PRNG_E_INVALID;
    SavedHeader hd;
    memcpy(&hd, host_buf, sizeof(hd));
    if (hd.magic != kMagic || hd.W != h->W || hd.m != h->g.m || hd.seed != h->seed ||
        hd.walk_len != h->g.walk_len || hd.burnin_len != h->g.burnin_len ||
        hd.variant != h->g.variant || hd.walker_base != h->o.walker_base ||
        hd.bit_source != h->o.bit_source)
        return PRNG_E_INVALID;
    // a resumed position must itself be reachable by the 32-bit draw cursor
    if (hd.N > kDrawLimit * h->W || hd.od_J0 > kDrawLimit) return PRNG_E_INVALID;
    if (h->od_open) return PRNG_E_STATE;
    return guard(h, [&] {
        CK(cudaDeviceSynchronize());
        const char *p = (const char *)host_buf + sizeof(hd);
        CK(cudaMemcpy(h->x, p, h->W * 4, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(h->y, p + h->W * 4, h->W * 4, cudaMemcpyHostToDevice));
        CK(cudaMemcpy(h->j, p + 2 * h->W * 4, h->W * 4, cudaMemcpyHostToDevice));
        h->N = hd.N;
        h->od_J0 = hd.od_J0;
        h->od_started = hd.od_started != 0;
        return PRNG_OK;
    });
}

static int epoch_begin_impl(prng_t *h, uint64_t active_walkers, const uint32_t *ids,
                            uint32_t draws, void *stream) {
    return guard(h, [&] {
        cudaStream_t s = (cudaStream_t)stream;
        const uint64_t J0 = h->od_started ? h->od_J0 : (h->N + h->W - 1) / h->W;
        if (J0 + draws > kDrawLimit) return PRNG_E_UNSUPPORTED;
        const int slot = h->od_slot ^ 1;
        // walkers [0, pf_hi) of this window were staged ahead (gg_epoch_prefeed)
        const bool pf = h->pf_valid && !ids && draws == 1 && h->pf_J0 == J0 &&
                        h->pf_slot == slot && active_walkers <= h->pf_pitch;
        h->pf_valid = false;
        const uint64_t pitch = pf ? h->pf_pitch : round_up(active_walkers, 32);
        const size_t bytes = (size_t)draws * h->R * pitch * 4;
        if (bytes > h->od_cap[slot] || (ids && active_walkers * 4 > h->od_wmap_cap[slot])) {
            CK(cudaEventSynchronize(h->od_free[slot]));
            if (bytes > h->od_cap[slot]) {
                if (h->od_buf[slot]) CK(cudaFree(h->od_buf[slot]));
                h->od_buf[slot] = nullptr;
                h->od_cap[slot] = 0;
                CK(cudaMalloc(&h->od_buf[slot], bytes));
                h->od_cap[slot] = bytes;
            }
            if (ids && active_walkers * 4 > h->od_wmap_cap[slot]) {
                if (h->od_wmap_buf[slot]) CK(cudaFree(h->od_wmap_buf[slot]));
                h->od_wmap_buf[slot] = nullptr;
                h->od_wmap_cap[slot] = 0;
                CK(cudaMalloc(&h->od_wmap_buf[slot], active_walkers * 4));
                h->od_wmap_cap[slot] = active_walkers * 4;
            }
        } else {
            // kernels of the epoch that last used this slot must be done with it
            CK(cudaStreamWaitEvent(h->copy_stream, h->od_free[slot], 0));
        }
        h->od_slot = slot;
        h->od_bits = h->od_buf[slot];
        h->od_wmap = nullptr;
        if (ids) {
            // the map travels with the bits (pageable source: the copy is staged by
            // the runtime, so the caller may reuse its array on return)
            CK(cudaMemcpyAsync(h->od_wmap_buf[slot], ids, active_walkers * 4,
                               cudaMemcpyHostToDevice, h->copy_stream));
            h->od_wmap = h->od_wmap_buf[slot];
            h->stats.h2d_bytes += active_walkers * 4;
        }
        // on-demand windows go past the CPU caches with paced streaming
        // stores (the consumer waits for the last chunk).  Windows >= 1 GB
        // (C4's 1.2 GB Monte Carlo epochs) used cached stores like bulk
        // streams until the shared-clock feed blocks; A/B hook
        // GG_FEED_EPOCH_CACHED=1 restores that.
        static const bool epoch_cached = getenv("GG_FEED_EPOCH_CACHED") != nullptr;
        const bool bursty = !epoch_cached || bytes < (1ull << 30);
        if (pf) {
            if (active_walkers > h->pf_hi) {  // the rest: walkers [pf_hi, active)
                const uint64_t lo = h->pf_hi, saved = h->o.walker_base;
                h->o.walker_base = saved + lo;
                stage_rows(h, 2 + h->R0 + h->R * J0, h->R, active_walkers - lo, h->od_bits + lo,
                           pitch, nullptr, true, true);
                h->o.walker_base = saved;
            }
        } else {
            stage_rows(h, 2 + h->R0 + h->R * J0, (uint64_t)draws * h->R, active_walkers,
                       h->od_bits, pitch, ids, bursty);
        }
        join_copies(h, s);
        h->od_J0 = J0;
        h->od_D = draws;
        h->od_Wv = active_walkers;
        h->od_pitch = pitch;
        h->od_open = true;
        h->od_started = true;
        return PRNG_OK;
    });
}

extern "C++" {
namespace gg {
double tl_now_us(prng_s *h) { return h && h->tl ? h->tl->now_us() : -1.0; }
void tl_host_span(prng_s *h, const char *kind, double a_us, double b_us) {
    if (h && h->tl && a_us >= 0.0) h->tl->host_span(kind, a_us, b_us);
}
cudaEvent_t tl_dev_begin(prng_s *h, cudaStream_t s) { return h && h->tl ? h->tl->begin(s) : nullptr; }
void tl_dev_end(prng_s *h, const char *kind, cudaEvent_t a, cudaStream_t s) {
    if (h && h->tl && a) h->tl->end(kind, a, s);
}

// Stage the next epoch's window ahead (one draw, walkers [0, hi), pitch
// `pitch` >= the next epoch's active count) while the current epoch's
// kernels run: list ranking knows the next round's active count only after
// its kernels, but not fewer than ~7/8 of this round's nodes survive.  The
// next prng_epoch_begin with draws = 1 and active <= pitch stages only the
// walkers above hi.  No effect on the numbers: a walker's bits at a draw are
// a pure function of (seed, walker, draw) (R9).
int epoch_prefeed(prng_t *h, uint64_t hi, uint64_t pitch) {
    if (!h || h->od_open || !h->od_started || hi == 0 || hi > pitch || pitch > round_up(h->W, 32))
        return PRNG_E_INVALID;
    return guard(h, [&] {
        const int slot = h->od_slot ^ 1;
        const uint64_t J0 = h->od_J0;
        const size_t bytes = (size_t)h->R * pitch * 4;
        if (bytes > h->od_cap[slot]) return PRNG_OK;  // not reserved: skip the prefeed
        CK(cudaStreamWaitEvent(h->copy_stream, h->od_free[slot], 0));
        stage_rows(h, 2 + h->R0 + h->R * J0, h->R, hi, h->od_buf[slot], pitch, nullptr, true);
        h->pf_valid = true;
        h->pf_slot = slot;
        h->pf_J0 = J0;
        h->pf_hi = hi;
        h->pf_pitch = pitch;
        return PRNG_OK;
    });
}
}  // namespace gg
}  // extern "C++"

int prng_epoch_begin(prng_t *h, uint64_t active_walkers, uint32_t draws, void *stream) {
    if (!h) return PRNG_E_INVALID;
    if (active_walkers == 0 || active_walkers > h->W || draws == 0) return PRNG_E_INVALID;
    if (h->od_open) return PRNG_E_STATE;
    return epoch_begin_impl(h, active_walkers, nullptr, draws, stream);
}

int prng_epoch_begin_list(prng_t *h, const uint32_t *walkers, uint64_t count, uint32_t draws,
                          void *stream) {
    if (!h || !walkers) return PRNG_E_INVALID;
    if (count == 0 || count > h->W || draws == 0) return PRNG_E_INVALID;
    for (uint64_t i = 0; i < count; i++)
        if (walkers[i] >= h->W) return PRNG_E_INVALID;
    if (h->od_open) return PRNG_E_STATE;
    return epoch_begin_impl(h, count, walkers, draws, stream);
}

int prng_epoch_reserve(prng_t *h, uint64_t active_walkers, uint32_t draws) {
    if (!h) return PRNG_E_INVALID;
    if (active_walkers == 0 || active_walkers > h->W || draws == 0) return PRNG_E_INVALID;
    if (h->od_open) return PRNG_E_STATE;
    return guard(h, [&] {
        const size_t bytes = (size_t)draws * h->R * round_up(active_walkers, 32) * 4;
        for (int slot = 0; slot < 2; slot++) {
            if (bytes <= h->od_cap[slot]) continue;
            CK(cudaEventSynchronize(h->od_free[slot]));
            if (h->od_buf[slot]) CK(cudaFree(h->od_buf[slot]));
            h->od_buf[slot] = nullptr;
            h->od_cap[slot] = 0;
            CK(cudaMalloc(&h->od_buf[slot], bytes));
            h->od_cap[slot] = bytes;
        }
        return PRNG_OK;
    });
}

int prng_epoch_end(prng_t *h, void *stream) {
    if (!h) return PRNG_E_INVALID;
    if (!h->od_open) return PRNG_E_STATE;
    if (cudaEventRecord(h->od_free[h->od_slot], (cudaStream_t)stream) != cudaSuccess) {
        h->poisoned = true;
        return PRNG_E_CUDA;
    }
    h->od_J0 += h->od_D;
    h->od_open = false;
    h->N = h->od_J0 * h->W;  // a later bulk fill starts with every walker at draw J0
    return PRNG_OK;
}

int prng_device_view(prng_t *h, void *view, size_t view_bytes) {
    if (!h || !view || view_bytes != sizeof(prng_view)) return PRNG_E_INVALID;
    if (!h->od_open) return PRNG_E_STATE;
    prng_view v{};
    v.bits = h->od_bits;
    v.wmap = h->od_wmap;
    v.x = h->x;
    v.y = h->y;
    v.j = h->j;
    v.flags = h->flags;
    v.pitch = h->od_pitch;
    v.m = h->g.m;
    v.J0 = (uint32_t)h->od_J0;
    v.D = h->od_D;
    v.Wv = (uint32_t)h->od_Wv;
    v.R = h->R;
    v.l = h->g.walk_len;
    v.log2m = h->log2m;
    v.pow2 = h->pow2;
    v.variant = h->g.variant;
    v.l0 = h->g.burnin_len;
    v.tab = h->walk_tab;
    memcpy(view, &v, sizeof(v));
    return PRNG_OK;
}

int prng_check(prng_t *h) {
    if (!h) return PRNG_E_INVALID;
    return guard(h, [&] {
        uint32_t f = 0;
        CK(cudaDeviceSynchronize());
        CK(cudaMemcpy(&f, h->flags, 4, cudaMemcpyDeviceToHost));
        if (f) {
            CK(cudaMemset(h->flags, 0, 4));
            return PRNG_E_OVERRUN;
        }
        return PRNG_OK;
    });
}

int prng_get_stats(prng_t *h, prng_stats *s) {
    if (!h || !s) return PRNG_E_INVALID;
    *s = h->stats;
    return PRNG_OK;
}

int prng_destroy(prng_t *h) {
    if (!h) return PRNG_OK;
    if (h->tl) {
        cudaSetDevice(h->o.device);
        h->tl->dump();
        delete h->tl;
        h->tl = nullptr;
    }
    free_all(h);
    delete h;
    return PRNG_OK;
}

}  // extern "C"

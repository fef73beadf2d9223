// Randomised list ranking with on-demand random numbers (§V,
// Alg.3 + Phases II/III of [3]).  C ABI: gg_list_rank (include/gg_apps.h).
//
// Phase I (Alg.3 ReduceList), one round per on-demand epoch:
//   lr_draw   : active slot i (walker i) calls prng_next; b(u) = bit 63 (R13)
//   lr_decide : u leaves iff b(u)=1, b(pred)=0, b(succ)=0, u not head/tail (R14)
//   lr_splice : splice u out; remember (pred, distance) for Phase III
//   gg::compact_flagged : stable single-pass compaction of the survivors
//               (compact.cu); the removed nodes of the round go straight to
//               the re-insertion log, the survivor count to mapped host
//               memory that the host polls while it stages the next round
//   repeat until active <= ceil(n / floor(log2 n)) (R15).  The host learns the
//   new active count each round and the feed supplies exactly that many draws
//   (on demand, instead of [3]'s upper-bound pre-generation).
// Phase II (Helman-JaJa [10]): splitters = head + nodes whose next draw is
//   < 2^64/64 (R18); each splitter walks its sublist (local offsets); suffix
//   sums over the splitter chain by pointer jumping; rank = prefix + local.
// Phase III: re-insert removed nodes in reverse round order,
//   rank(u) = rank(pred at removal) + distance at removal.
#include <chrono>
#include <cmath>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <map>
#include <memory>
#include <mutex>
#include <vector>

#include <atomic>
#include <thread>

#include <cuda_runtime.h>

#include "gg_apps.h"
#include "gg_internal.h"
#include "prng.h"
#include "prng_device.cuh"

namespace {

struct Fail {
    int rc;
};
#define LCK(call)                                              \
    do {                                                       \
        cudaError_t _e = (call);                               \
        if (_e != cudaSuccess) throw Fail{PRNG_E_CUDA};        \
    } while (0)
#define LRC(call)                                              \
    do {                                                       \
        int _r = (call);                                       \
        if (_r != PRNG_OK) throw Fail{_r};                     \
    } while (0)

__global__ void lr_init(int64_t n, int32_t *act, int32_t *w, int32_t *rr, int32_t *spl) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= n) return;
    act[i] = (int32_t)i;  // A_0 = node ids in order
    w[i] = 1;             // links from i to succ(i)
    if (rr) rr[i] = -1;
    if (spl) spl[i] = 0;
}

__global__ void lr_find_tail(int64_t n, const int32_t *succ, int32_t *tail) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < n && succ[i] < 0) *tail = (int32_t)i;
}

// Alg.3 l.6-7: temp = getnextrand(); b(u) = bit 63 of temp.
// MODE: PRNG_WALK_L64 for the paper's generator (only that walk compiled in),
// PRNG_WALK_AUTO (run-time dispatch) for other graph parameters.
template <int MODE>
__global__ void __launch_bounds__(128) lr_draw(const __grid_constant__ prng_view v,
                                               const int32_t *act, int64_t A, uint8_t *bit) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= A) return;
    prng_state st = prng_state_load(&v, (uint32_t)i);
    const uint64_t z = prng_next<MODE>(&st, &v);
    prng_state_store(&v, &st);
    bit[act[i]] = (uint8_t)(z >> 63);
}

// Alg.3 l.8-9 on the bits of this round (no list change yet).
__global__ void lr_decide(const int32_t *act, int64_t A, const uint8_t *bit, const int32_t *pred,
                          const int32_t *succ, int32_t head, int32_t tail, uint8_t *keep) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= A) return;
    const int32_t u = act[i];
    bool rm = false;
    if (u != head && u != tail) rm = bit[u] && !bit[pred[u]] && !bit[succ[u]];
    keep[i] = rm ? 0 : 1;
}

// Alg.3 l.10: remove with book-keeping.  No two removed nodes are adjacent,
// so every written field has exactly one writer.
__global__ void lr_splice(const int32_t *act, int64_t A, const uint8_t *keep, int32_t *pred,
                          int32_t *succ, int32_t *w, int32_t *rem_pred, int32_t *rem_dist,
                          int32_t *rr, int32_t round) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= A || keep[i]) return;
    const int32_t u = act[i], p = pred[u], s = succ[u];
    rem_pred[u] = p;
    rem_dist[u] = w[p];
    w[p] += w[u];
    succ[p] = s;
    pred[s] = p;
    if (rr) rr[u] = round;
}

// Phase II splitter choice (R18).
template <int MODE>
__global__ void __launch_bounds__(128) lr_splitter_draw(const __grid_constant__ prng_view v,
                                                        const int32_t *act, int64_t A,
                                                        int32_t head, uint8_t *spl_node,
                                                        uint8_t *spl_slot, int32_t *spl_out) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= A) return;
    prng_state st = prng_state_load(&v, (uint32_t)i);
    const uint64_t z = prng_next<MODE>(&st, &v);
    prng_state_store(&v, &st);
    const int32_t u = act[i];
    const uint8_t s = (u == head || (z >> 58) == 0) ? 1 : 0;
    spl_node[u] = s;
    spl_slot[i] = s;
    if (spl_out) spl_out[u] = s;
}

__global__ void lr_splitter_index(const int32_t *spl, int64_t ns, int32_t *spl_idx) {
    const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (k < ns) spl_idx[spl[k]] = (int32_t)k;
}

// Sublist walk: splitter k in [k0, k1) follows succ to the next splitter.
__global__ void lr_sublist(const int32_t *spl, int64_t k0, int64_t k1, const int32_t *succ,
                           const int32_t *w, const uint8_t *spl_node, const int32_t *spl_idx,
                           int32_t *local, int32_t *sub, int32_t *len, int32_t *nextk) {
    const int64_t k = k0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= k1) return;
    int32_t v = spl[k], off = 0;
    for (;;) {
        local[v] = off;
        sub[v] = (int32_t)k;
        off += w[v];
        const int32_t nx = succ[v];
        if (nx < 0 || spl_node[nx]) {
            len[k] = off;
            nextk[k] = nx < 0 ? -1 : spl_idx[nx];
            return;
        }
        v = nx;
    }
}

// One pointer-jumping step of suffix sums over the splitter chain (Wyllie).
__global__ void lr_jump(int64_t ns, const int32_t *val_in, const int32_t *nxt_in, int32_t *val_out,
                        int32_t *nxt_out) {
    const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= ns) return;
    const int32_t nx = nxt_in[k];
    if (nx >= 0) {
        val_out[k] = val_in[k] + val_in[nx];
        nxt_out[k] = nxt_in[nx];
    } else {
        val_out[k] = val_in[k];
        nxt_out[k] = -1;
    }
}

// rank = (total - suffix of own sublist) + local offset, for nodes whose
// sublist this rank walked (sub >= 0); slot_rank[i] gets the same value (0
// for nodes of other ranks) for the cross-rank sum.
__global__ void lr_fixup(const int32_t *act, int64_t A, const int32_t *sub, const int32_t *local,
                         const int32_t *suffix, const int32_t *spl_idx, int32_t head,
                         int32_t *rank, int32_t *slot_rank) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= A) return;
    const int32_t v = act[i];
    const int32_t sb = sub[v];
    int32_t r = 0;
    if (sb >= 0) {
        const int32_t total = suffix[spl_idx[head]];
        r = total - suffix[sb] + local[v];
        rank[v] = r;
    }
    if (slot_rank) slot_rank[i] = r;
}

// Rebuild the full splitter tables from the allgathered per-rank chunks:
// rank q contributed splitters [q*ns/G, (q+1)*ns/G) at offset q*chunk.
__global__ void lr_unpack(const int2 *recv, int64_t ns, int world, int64_t chunk, int32_t *len,
                          int32_t *nextk) {
    const int64_t k = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (k >= ns) return;
    int q = (int)((k * world) / ns);
    while (q + 1 < world && (q + 1) * ns / world <= k) q++;
    while (q > 0 && q * ns / world > k) q--;
    const int64_t k0 = q * ns / world;
    const int2 rec = recv[q * chunk + (k - k0)];
    len[k] = rec.x;
    nextk[k] = rec.y;
}

__global__ void lr_pack(const int32_t *len, const int32_t *nextk, int64_t k0, int64_t k1,
                        int2 *send) {
    const int64_t k = k0 + (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (k < k1) send[k - k0] = make_int2(len[k], nextk[k]);
}

__global__ void lr_scatter_slot_rank(const int32_t *act, int64_t A, const int32_t *slot_rank,
                                     int32_t *rank) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i < A) rank[act[i]] = slot_rank[i];
}

__global__ void lr_reinsert(const int32_t *list, int64_t cnt, const int32_t *rem_pred,
                            const int32_t *rem_dist, int32_t *rank) {
    const int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
    if (i >= cnt) return;
    const int32_t u = list[i];
    rank[u] = rank[rem_pred[u]] + rem_dist[u];
}

inline unsigned nblk(int64_t n, int t = 256) { return (unsigned)((n + t - 1) / t); }

// Mapped pinned 8-byte slots the compaction kernel writes its count into
// (one per concurrent gg_list_rank call; allocated in blocks, never freed).
struct CountSlot {
    volatile uint64_t *p = nullptr;
    CountSlot() {
        std::lock_guard<std::mutex> lk(mu());
        if (free_list().empty()) {
            void *blk = nullptr;
            if (cudaHostAlloc(&blk, 64 * 64, cudaHostAllocMapped | cudaHostAllocPortable) !=
                cudaSuccess)
                throw Fail{PRNG_E_NOMEM};
            for (int i = 0; i < 64; i++)
                free_list().push_back((volatile uint64_t *)((char *)blk + 64 * i));
        }
        p = free_list().back();
        free_list().pop_back();
    }
    ~CountSlot() {
        std::lock_guard<std::mutex> lk(mu());
        free_list().push_back(p);
    }
    static std::mutex &mu() {
        static std::mutex m;
        return m;
    }
    static std::vector<volatile uint64_t *> &free_list() {
        static std::vector<volatile uint64_t *> v;
        return v;
    }
};

std::atomic<uint32_t> g_tag{1};

// Wait until the compaction kernel tagged `tag` has published its count
// (polling mapped host memory, no stream synchronisation); CUDA errors on the
// stream end the wait.
int32_t wait_count(volatile uint64_t *slot, uint32_t tag, cudaStream_t s) {
    for (uint32_t spin = 0;; spin++) {
        const uint64_t v = *slot;
        if ((uint32_t)(v >> 32) == tag) return (int32_t)(uint32_t)v;
        if ((spin & 255u) == 255u) {
            const cudaError_t e = cudaStreamQuery(s);
            if (e != cudaSuccess && e != cudaErrorNotReady) throw Fail{PRNG_E_CUDA};
            if (e == cudaSuccess) {
                const uint64_t w = *slot;  // the stream is done: the value must be there
                if ((uint32_t)(w >> 32) == tag) return (int32_t)(uint32_t)w;
                throw Fail{PRNG_E_CUDA};
            }
            std::this_thread::yield();
        }
    }
}

}  // namespace

// Stream-ordered scratch pool of this library, one per device, that keeps its
// memory between calls (release threshold = max): the default pool returns
// freed memory to the driver at every synchronisation, and re-mapping the
// ~0.7 GB of C3 scratch made repeated calls' wall time erratic.
cudaMemPool_t gg::scratch_pool() {
    static std::mutex mu;
    static std::map<int, cudaMemPool_t> pools;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) return nullptr;
    std::lock_guard<std::mutex> lk(mu);
    auto it = pools.find(dev);
    if (it != pools.end()) return it->second;
    cudaMemPoolProps props{};
    props.allocType = cudaMemAllocationTypePinned;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    cudaMemPool_t p = nullptr;
    if (cudaMemPoolCreate(&p, &props) != cudaSuccess) return nullptr;
    uint64_t thr = UINT64_MAX;
    cudaMemPoolSetAttribute(p, cudaMemPoolAttrReleaseThreshold, &thr);
    pools[dev] = p;
    return p;
}

extern "C" int gg_list_rank(prng_t *h, int64_t n, const int32_t *succ, const int32_t *pred,
                            int64_t head, int32_t *rank, int32_t *removed_round,
                            int32_t *is_splitter, int64_t *info, const gg_collective *coll,
                            void *stream) {
    if (!h || n <= 0 || !succ || !pred || !rank || head < 0 || head >= n) return PRNG_E_INVALID;
    const int world = coll ? coll->world : 1;
    const int me = coll ? coll->rank : 0;
    if (world < 1 || me < 0 || me >= world ||
        (world > 1 && (!coll->allgather || !coll->allreduce_i32)))
        return PRNG_E_INVALID;
    if (n > (1ll << 24)) return PRNG_E_UNSUPPORTED;
    for (const void *p : {(const void *)succ, (const void *)pred, (const void *)rank,
                          (const void *)removed_round, (const void *)is_splitter})
        if (((uintptr_t)p % 4) != 0) return PRNG_E_INVALID;
    cudaStream_t s = (cudaStream_t)stream;
    std::vector<void *> bufs;
    cudaMemPool_t pool = gg::scratch_pool();
    if (!pool) return PRNG_E_CUDA;
    auto alloc = [&](size_t bytes) -> void * {
        void *p = nullptr;
        LCK(cudaMallocFromPoolAsync(&p, bytes ? bytes : 1, pool, s));
        bufs.push_back(p);
        return p;
    };
    int rc = PRNG_OK;
    // held until the stream is known idle: a compaction kernel still in
    // flight after a failure must not write into a slot another call owns
    std::unique_ptr<CountSlot> slot_owner;
    try {
        cudaEvent_t ev[4];
        for (auto &e : ev) LCK(cudaEventCreate(&e));
        LCK(cudaEventRecord(ev[0], s));
        const size_t n4 = (size_t)n * 4;
        int32_t *d_succ = (int32_t *)alloc(n4), *d_pred = (int32_t *)alloc(n4);
        int32_t *w = (int32_t *)alloc(n4), *rem_pred = (int32_t *)alloc(n4);
        int32_t *rem_dist = (int32_t *)alloc(n4), *act = (int32_t *)alloc(n4);
        int32_t *act2 = (int32_t *)alloc(n4), *rem_log = (int32_t *)alloc(n4);
        uint8_t *bit = (uint8_t *)alloc(n), *keep = (uint8_t *)alloc(n);
        int32_t *d_num = (int32_t *)alloc(8);
        LCK(cudaMemcpyAsync(d_succ, succ, n4, cudaMemcpyDeviceToDevice, s));
        LCK(cudaMemcpyAsync(d_pred, pred, n4, cudaMemcpyDeviceToDevice, s));
        lr_init<<<nblk(n), 256, 0, s>>>(n, act, w, removed_round, is_splitter);
        // the tail is the node whose succ is -1
        LCK(cudaMemsetAsync(d_num, 0xFF, 8, s));
        lr_find_tail<<<nblk(n), 256, 0, s>>>(n, d_succ, d_num + 1);
        int32_t tail = -1;
        LCK(cudaMemcpyAsync(&tail, d_num + 1, 4, cudaMemcpyDeviceToHost, s));
        void *tmp = alloc(gg::compact_scratch_bytes(n));
        slot_owner.reset(new CountSlot());
        CountSlot &slot = *slot_owner;
        LCK(cudaStreamSynchronize(s));
        if (tail < 0) throw Fail{PRNG_E_INVALID};

        int64_t L = 0;
        while ((1ll << (L + 1)) <= n) L++;
        if (L == 0) L = 1;
        const int64_t target = (n + L - 1) / L;
        int64_t A = n, rounds = 0, draws = 0, log_off = 0;
        std::vector<int64_t> round_off, round_cnt;
        prng_view view;
        // both window slots sized for the first (largest) round: the slot
        // parity flips between calls (rounds + 1 epochs per call)
        LRC(prng_epoch_reserve(h, (uint64_t)n, 1));
        // ---------------- Phase I
        static const bool trace = getenv("GG_LR_TRACE") != nullptr;
        while (A > target && rounds < 1000) {
            auto tr0 = std::chrono::steady_clock::now();
            const double tb0 = gg::tl_now_us(h);
            LRC(prng_epoch_begin(h, (uint64_t)A, 1, s));
            gg::tl_host_span(h, "lr.begin", tb0, gg::tl_now_us(h));
            cudaEvent_t tk0 = gg::tl_dev_begin(h, s);
            auto tr1 = std::chrono::steady_clock::now();
            static const bool fine = trace && atoi(getenv("GG_LR_TRACE")) >= 2;
            auto sync_t = [&](const char *what, std::chrono::steady_clock::time_point &t) {
                if (!fine) return;
                cudaStreamSynchronize(s);
                auto now = std::chrono::steady_clock::now();
                fprintf(stderr, "   %s %.3f ms\n", what,
                        std::chrono::duration<double, std::milli>(now - t).count());
                t = now;
            };
            auto tq = std::chrono::steady_clock::now();
            sync_t("copy-wait", tq);
            LRC(prng_device_view(h, &view, sizeof(view)));
            if (prng_walk_mode(&view) == PRNG_WALK_L64)
                lr_draw<PRNG_WALK_L64><<<nblk(A, 128), 128, 0, s>>>(view, act, A, bit);
            else
                lr_draw<PRNG_WALK_AUTO><<<nblk(A, 128), 128, 0, s>>>(view, act, A, bit);
            LRC(prng_epoch_end(h, s));
            sync_t("draw", tq);
            draws += A;
            lr_decide<<<nblk(A), 256, 0, s>>>(act, A, bit, d_pred, d_succ, (int32_t)head, tail, keep);
            lr_splice<<<nblk(A), 256, 0, s>>>(act, A, keep, d_pred, d_succ, w, rem_pred, rem_dist,
                                              removed_round, (int32_t)rounds);
            sync_t("decide+splice", tq);
            const uint32_t tag = g_tag.fetch_add(1);
            LCK(gg::compact_flagged(act, keep, A, act2, rem_log + log_off, d_num, slot.p, tag, tmp,
                                    s));
            sync_t("partition", tq);
            gg::tl_dev_end(h, "lr.kernels", tk0, s);
            // While this round's kernels run, stage the next round's bits for the
            // slots that will most likely stay active: an interior node is removed
            // with probability 1/8 (Alg.3 l.8-9), so the survivors are ~7/8 A with
            // a standard deviation of sqrt(7A)/8.  Staging up to 7/8 A + 3 sd
            // (capped at this round's pitch, an upper bound) leaves no remainder
            // to stage after the count is known in all but ~0.1% of rounds, at
            // ~3 sd x 24 B of unused bits (~40 KB at A = 2^24); a remainder, when
            // there is one, is staged by the next prng_epoch_begin.  Bits are a
            // pure function of (seed, slot, round), so the numbers do not depend
            // on this bound.  GG_LR_PREFEED=0: off; =2: the round-1 bound 7/8 A -
            // 8 sd (never more than the survivors; one remainder every round).
            static const int prefeed_mode =
                getenv("GG_LR_PREFEED") ? atoi(getenv("GG_LR_PREFEED")) : 1;
            if (prefeed_mode != 0 && A > 4096) {
                const double sd = std::sqrt(7.0 * (double)A) / 8.0;
                const int64_t lo = prefeed_mode == 2
                                       ? (int64_t)(0.875 * (double)A - 8.0 * sd)
                                       : std::min<int64_t>(A, (int64_t)(0.875 * (double)A + 3.0 * sd));
                const double tp0 = gg::tl_now_us(h);
                if (lo > 0) LRC(gg::epoch_prefeed(h, (uint64_t)lo, ((uint64_t)A + 31) / 32 * 32));
                gg::tl_host_span(h, "lr.prefeed", tp0, gg::tl_now_us(h));
            }
            const double tw0 = gg::tl_now_us(h);
            const int32_t kept = wait_count(slot.p, tag, s);
            gg::tl_host_span(h, "lr.wait", tw0, gg::tl_now_us(h));
            if (trace) {
                auto tr2 = std::chrono::steady_clock::now();
                fprintf(stderr, "[lr] round %ld A=%ld feed+enqueue %.3f ms, kernels+sync %.3f ms\n",
                        (long)rounds, (long)A,
                        std::chrono::duration<double, std::milli>(tr1 - tr0).count(),
                        std::chrono::duration<double, std::milli>(tr2 - tr1).count());
            }
            const int64_t gone = A - kept;
            round_off.push_back(log_off);
            round_cnt.push_back(gone);
            log_off += gone;
            std::swap(act, act2);
            A = kept;
            rounds++;
        }
        LCK(cudaEventRecord(ev[1], s));
        // ---------------- Phase II
        uint8_t *spl_node = bit;  // reuse: bits of Phase I are dead
        LRC(prng_epoch_begin(h, (uint64_t)A, 1, s));
        LRC(prng_device_view(h, &view, sizeof(view)));
        LCK(cudaMemsetAsync(spl_node, 0, n, s));
        if (prng_walk_mode(&view) == PRNG_WALK_L64)
            lr_splitter_draw<PRNG_WALK_L64><<<nblk(A, 128), 128, 0, s>>>(
                view, act, A, (int32_t)head, spl_node, keep, is_splitter);
        else
            lr_splitter_draw<PRNG_WALK_AUTO><<<nblk(A, 128), 128, 0, s>>>(
                view, act, A, (int32_t)head, spl_node, keep, is_splitter);
        LRC(prng_epoch_end(h, s));
        draws += A;
        const uint32_t tag2 = g_tag.fetch_add(1);
        LCK(gg::compact_flagged(act, keep, A, act2, nullptr, d_num, slot.p, tag2, tmp, s));
        const int32_t ns = wait_count(slot.p, tag2, s);
        int32_t *spl = act2;
        int32_t *spl_idx = (int32_t *)alloc(n4);
        int32_t *local = (int32_t *)alloc(n4), *sub = (int32_t *)alloc(n4);
        int32_t *va = (int32_t *)alloc((size_t)ns * 4), *na = (int32_t *)alloc((size_t)ns * 4);
        int32_t *vb = (int32_t *)alloc((size_t)ns * 4), *nb = (int32_t *)alloc((size_t)ns * 4);
        LCK(cudaMemsetAsync(sub, 0xFF, n4, s));  // -1: not in a sublist walked here
        lr_splitter_index<<<nblk(ns), 256, 0, s>>>(spl, ns, spl_idx);
        // this rank's share of the sublists (all of them on one GPU)
        const int64_t k0 = (int64_t)me * ns / world, k1 = (int64_t)(me + 1) * ns / world;
        if (k1 > k0)
            lr_sublist<<<nblk(k1 - k0, 128), 128, 0, s>>>(spl, k0, k1, d_succ, w, spl_node, spl_idx,
                                                         local, sub, va, na);
        int32_t *slot_rank = nullptr;
        if (world > 1) {
            // splitter exchange: one allgather of (sublist length, next splitter)
            const int64_t chunk = (ns + world - 1) / world;
            int2 *send = (int2 *)alloc((size_t)chunk * 8);
            int2 *recv = (int2 *)alloc((size_t)chunk * 8 * world);
            if (k1 > k0) lr_pack<<<nblk(k1 - k0), 256, 0, s>>>(va, na, k0, k1, send);
            LCK(cudaStreamSynchronize(s));
            if (coll->allgather(coll->ctx, send, recv, (size_t)chunk * 8) != 0)
                throw Fail{PRNG_E_CUDA};
            lr_unpack<<<nblk(ns), 256, 0, s>>>(recv, ns, world, chunk, va, na);
            slot_rank = (int32_t *)alloc((size_t)A * 4);
        }
        int iters = 0;
        while ((1ll << iters) < (int64_t)ns) iters++;
        for (int it = 0; it <= iters; it++) {
            lr_jump<<<nblk(ns), 256, 0, s>>>(ns, va, na, vb, nb);
            std::swap(va, vb);
            std::swap(na, nb);
        }
        lr_fixup<<<nblk(A), 256, 0, s>>>(act, A, sub, local, va, spl_idx, (int32_t)head, rank,
                                        slot_rank);
        if (world > 1) {
            // every reduced node was ranked by exactly one rank: sum the slot arrays
            LCK(cudaStreamSynchronize(s));
            if (coll->allreduce_i32(coll->ctx, slot_rank, (size_t)A) != 0) throw Fail{PRNG_E_CUDA};
            lr_scatter_slot_rank<<<nblk(A), 256, 0, s>>>(act, A, slot_rank, rank);
        }
        LCK(cudaEventRecord(ev[2], s));
        // ---------------- Phase III
        for (int64_t r = rounds - 1; r >= 0; r--) {
            const int64_t cnt = round_cnt[r];
            if (cnt)
                lr_reinsert<<<nblk(cnt), 256, 0, s>>>(rem_log + round_off[r], cnt, rem_pred,
                                                      rem_dist, rank);
        }
        LCK(cudaEventRecord(ev[3], s));
        LCK(cudaGetLastError());
        LCK(cudaEventSynchronize(ev[3]));
        if (info) {
            float t1, t2, t3;
            LCK(cudaEventElapsedTime(&t1, ev[0], ev[1]));
            LCK(cudaEventElapsedTime(&t2, ev[1], ev[2]));
            LCK(cudaEventElapsedTime(&t3, ev[2], ev[3]));
            info[0] = rounds;
            info[1] = A;
            info[2] = ns;
            info[3] = draws;
            info[4] = (int64_t)(t1 * 1000.0f);
            info[5] = (int64_t)(t2 * 1000.0f);
            info[6] = (int64_t)(t3 * 1000.0f);
            info[7] = (int64_t)round_cnt.size();
        }
        for (auto &e : ev) cudaEventDestroy(e);
    } catch (const Fail &f) {
        rc = f.rc;
    }
    for (void *p : bufs) cudaFreeAsync(p, s);
    const bool idle = cudaStreamSynchronize(s) == cudaSuccess;
    if (rc == PRNG_OK && !idle) rc = PRNG_E_CUDA;
    if (!idle) slot_owner.release();  // never reuse a slot a kernel may still write
    return rc;
}

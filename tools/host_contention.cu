// Diagnostic (tool): pinned H2D rate while host threads stream-store into
// other pinned memory -- the FEED's regime (feed threads write seed bits with
// non-temporal stores while the copy engine reads earlier chunks).
//
//   nvcc -O3 -std=c++17 -Xcompiler -mavx512f,-pthread -o tools/host_contention tools/host_contention.cu
//   tools/host_contention [threads ...]        (default 0 2 4 8 12 16)
//
// For each writer-thread count T: T threads write a private 256 MB pinned
// buffer each, over and over, with 64-byte non-temporal stores, while the
// main thread times 32 H2D copies of 256 MB (CUDA events); the writers'
// rate is their bytes stored over the same window.  Prints one JSON
// object: per T the H2D GB/s and the writers' aggregate GB/s; their sum is
// the host memory traffic the two sustain together.
#include <immintrin.h>

#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <thread>
#include <vector>

#include <cuda_runtime.h>

#define CK(x)                                                                    \
    do {                                                                         \
        cudaError_t e_ = (x);                                                    \
        if (e_ != cudaSuccess) {                                                 \
            fprintf(stderr, "%s: %s\n", #x, cudaGetErrorString(e_));             \
            exit(1);                                                             \
        }                                                                        \
    } while (0)

static constexpr size_t kBuf = 256ull << 20;

int main(int argc, char **argv) {
    std::vector<int> counts;
    for (int i = 1; i < argc; i++) counts.push_back(atoi(argv[i]));
    if (counts.empty()) counts = {0, 2, 4, 8, 12, 16};
    int maxt = 0;
    for (int t : counts) maxt = t > maxt ? t : maxt;
    void *src, *dst;
    CK(cudaMallocHost(&src, kBuf));
    CK(cudaMalloc(&dst, kBuf));
    memset(src, 1, kBuf);
    std::vector<void *> wbuf(maxt);
    for (int i = 0; i < maxt; i++) {
        CK(cudaMallocHost(&wbuf[i], kBuf));
        memset(wbuf[i], 0, kBuf);
    }
    cudaStream_t s;
    CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    cudaEvent_t e0, e1;
    CK(cudaEventCreate(&e0));
    CK(cudaEventCreate(&e1));
    for (int r = 0; r < 4; r++) CK(cudaMemcpyAsync(dst, src, kBuf, cudaMemcpyHostToDevice, s));
    CK(cudaStreamSynchronize(s));
    printf("{\"buffer_mb\": %zu, \"runs\": [", kBuf >> 20);
    for (size_t ci = 0; ci < counts.size(); ci++) {
        const int T = counts[ci];
        std::atomic<bool> stop{false};
        std::atomic<uint64_t> progress{0};  // bytes stored, counted per 4 MB block
        std::vector<std::thread> th;
        for (int i = 0; i < T; i++)
            th.emplace_back([&, i] {
                __m512i v = _mm512_set1_epi64(0x5EED0000 + i);
                const __m512i inc = _mm512_set1_epi64(1);
                constexpr size_t kBlk = 4u << 20;
                while (!stop.load(std::memory_order_relaxed)) {
                    for (size_t off = 0; off < kBuf && !stop.load(std::memory_order_relaxed); off += kBlk) {
                        __m512i *p = (__m512i *)((char *)wbuf[i] + off);
                        for (size_t k = 0; k < kBlk / 64; k++) {
                            _mm512_stream_si512(p + k, v);
                            v = _mm512_add_epi64(v, inc);
                        }
                        progress.fetch_add(kBlk, std::memory_order_relaxed);
                    }
                    _mm_sfence();
                }
            });
        std::this_thread::sleep_for(std::chrono::milliseconds(100));
        const auto t0 = std::chrono::steady_clock::now();
        const uint64_t p0 = progress.load();
        CK(cudaEventRecord(e0, s));
        const int reps = 32;
        for (int r = 0; r < reps; r++) CK(cudaMemcpyAsync(dst, src, kBuf, cudaMemcpyHostToDevice, s));
        CK(cudaEventRecord(e1, s));
        CK(cudaEventSynchronize(e1));
        const uint64_t p1 = progress.load();
        const auto t1 = std::chrono::steady_clock::now();
        stop = true;
        for (auto &x : th) x.join();
        float ms;
        CK(cudaEventElapsedTime(&ms, e0, e1));
        const double h2d = reps * (double)kBuf / (ms / 1e3) / 1e9;
        const double wgbs = (double)(p1 - p0) / std::chrono::duration<double>(t1 - t0).count() / 1e9;
        printf("%s{\"writer_threads\": %d, \"h2d_gbs\": %.2f, \"writers_gbs\": %.2f}", ci ? ", " : "", T,
               h2d, wgbs);
        fflush(stdout);
    }
    printf("]}\n");
    return 0;
}

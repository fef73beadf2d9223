/*
 * examples/c_consumer.cu — using the library from C/CUDA without Python.
 *
 * Links only libggprng.so and includes only the public headers:
 *   include/prng.h         host C ABI (prng_create / prng_fill / epochs)
 *   include/prng_device.cuh header-only device API (prng_next, Alg.2)
 * It (1) bulk-fills 4 numbers per walker (prng_fill, R11 order), (2) opens an
 * on-demand epoch and runs its OWN kernel in which thread t calls prng_next
 * (t % 3) + 1 times on walker t — the "any thread, any time, unknown count"
 * use the paper targets (§I-A, §III), then (3) prints, one per
 * line, "bulk t j value" and "od t i value" for a few walkers, which
 * tests/test_gpu_example.py compares with the oracle.
 *
 *   usage: c_consumer <walkers> <seed_hex>
 */
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdlib.h>

#include "prng.h"
#include "prng_device.cuh"

#define CHECK(call)                                                                     \
    do {                                                                                \
        int rc_ = (call);                                                               \
        if (rc_ != PRNG_OK) {                                                           \
            fprintf(stderr, "%s failed: %s\n", #call, prng_strerror(rc_));              \
            return 1;                                                                   \
        }                                                                               \
    } while (0)

__global__ void user_kernel(const __grid_constant__ prng_view v, uint32_t walkers,
                            unsigned long long *out) {
    const uint32_t t = blockIdx.x * blockDim.x + threadIdx.x;
    if (t >= walkers) return;
    prng_state st = prng_state_load(&v, t);
    const uint32_t calls = t % 3u + 1u;  // data-dependent demand
    for (uint32_t i = 0; i < calls; i++) out[(size_t)t * 3 + i] = prng_next(&st);  // north_star's prng_next(&state)
    prng_state_store(&st);
}

int main(int argc, char **argv) {
    const uint32_t W = argc > 1 ? (uint32_t)strtoul(argv[1], NULL, 0) : 1000;
    const uint64_t seed = argc > 2 ? strtoull(argv[2], NULL, 16) : 0x5EED;
    prng_graph_params g;
    prng_default_params(&g);  // m = 2^32, degree 7, l = l0 = 64
    prng_t *h = NULL;
    CHECK(prng_create(&h, &g, W, seed, NULL));

    unsigned long long *d_bulk = NULL, *d_od = NULL;
    cudaMalloc(&d_bulk, sizeof(unsigned long long) * W * 4);
    cudaMalloc(&d_od, sizeof(unsigned long long) * W * 3);
    cudaMemset(d_od, 0, sizeof(unsigned long long) * W * 3);
    CHECK(prng_fill(h, d_bulk, (uint64_t)W * 4, PRNG_FMT_U64, NULL));

    CHECK(prng_epoch_begin(h, W, 3, NULL));
    prng_view v;
    CHECK(prng_device_view(h, &v, sizeof(v)));
    user_kernel<<<(W + 127) / 128, 128>>>(v, W, d_od);
    CHECK(prng_epoch_end(h, NULL));
    cudaDeviceSynchronize();
    if (cudaGetLastError() != cudaSuccess) return 2;
    CHECK(prng_check(h));

    unsigned long long *bulk = (unsigned long long *)malloc(sizeof(unsigned long long) * W * 4);
    unsigned long long *od = (unsigned long long *)malloc(sizeof(unsigned long long) * W * 3);
    cudaMemcpy(bulk, d_bulk, sizeof(unsigned long long) * W * 4, cudaMemcpyDeviceToHost);
    cudaMemcpy(od, d_od, sizeof(unsigned long long) * W * 3, cudaMemcpyDeviceToHost);
    const uint32_t sample[] = {0, 1, 2, W / 2, W - 1};
    for (int s = 0; s < 5; s++) {
        const uint32_t t = sample[s];
        for (uint32_t j = 0; j < 4; j++) printf("bulk %u %u 0x%016llx\n", t, j, bulk[(size_t)j * W + t]);
        for (uint32_t i = 0; i < t % 3u + 1u; i++) printf("od %u %u 0x%016llx\n", t, i, od[(size_t)t * 3 + i]);
    }
    CHECK(prng_destroy(h));
    cudaFree(d_bulk);
    cudaFree(d_od);
    free(bulk);
    free(od);
    return 0;
}

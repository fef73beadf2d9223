"""Fig. 6 analogue (tool; §IV-A "Comparison with rand()").

    python tools/fig6.py [out.json]

The paper runs its generator on a multicore CPU alone and compares the time
to produce N numbers with glibc rand() (Fig. 6), then proposes using the CPU
generator "in the place of rand()" as the hybrid's bit source.  Measured here
on the GPU box's host:
  * glibc rand(): N calls in one thread (rand() holds a lock; the paper's
    "CPU Rand Time" is single-threaded), plus rand_r on all cores;
  * the generator on the host (the feed's bit_source 3 code path, R23):
    64-bit labels per second on one feed thread and on all of them, timed
    inside the feed thread pool during prng_prefetch;
  * the GPU generator fed by it end to end (prng_fill, bits streamed from the
    host walk): numbers/s, i.e. the hybrid with the CPU generator as FEED.
"""
import ctypes
import json
import os
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

RAND_C = r'''
#include <stdlib.h>
#include <stdint.h>
#include <pthread.h>
uint64_t rand_loop(uint64_t n) { uint64_t acc = 0; for (uint64_t i = 0; i < n; i++) acc += (uint64_t)rand(); return acc; }
typedef struct { uint64_t n; unsigned s; uint64_t acc; } job_t;
static void *rr(void *p) { job_t *j = (job_t *)p; for (uint64_t i = 0; i < j->n; i++) j->acc += (uint64_t)rand_r(&j->s); return 0; }
uint64_t rand_r_threads(uint64_t n, int threads) {
  pthread_t th[256]; job_t jb[256]; uint64_t acc = 0;
  for (int i = 0; i < threads; i++) { jb[i].n = n / threads; jb[i].s = 1234u + i; jb[i].acc = 0; pthread_create(&th[i], 0, rr, &jb[i]); }
  for (int i = 0; i < threads; i++) { pthread_join(th[i], 0); acc += jb[i].acc; }
  return acc;
}
'''


def main():
    res = {}
    d = tempfile.mkdtemp()
    src, so = os.path.join(d, "r.c"), os.path.join(d, "r.so")
    with open(src, "w") as f:
        f.write(RAND_C)
    subprocess.check_call(["gcc", "-O2", "-shared", "-fPIC", "-pthread", "-o", so, src])
    lib = ctypes.CDLL(so)
    lib.rand_loop.restype = ctypes.c_uint64
    lib.rand_loop.argtypes = [ctypes.c_uint64]
    lib.rand_r_threads.restype = ctypes.c_uint64
    lib.rand_r_threads.argtypes = [ctypes.c_uint64, ctypes.c_int]
    n = 200_000_000
    t = time.perf_counter()
    lib.rand_loop(n)
    dt = time.perf_counter() - t
    cores = os.cpu_count() or 1
    res["glibc_rand_1thread"] = {"numbers_per_s": n / dt, "bits_per_number": 31}
    t = time.perf_counter()
    lib.rand_r_threads(n * 4, cores)
    dt2 = time.perf_counter() - t
    res["glibc_rand_r_all_threads"] = {"numbers_per_s": n * 4 / dt2, "threads": cores}

    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W = 1 << 18
    for threads in (1, cores):
        g = Generator(walkers=W, seed=0x5EED0006, bit_source=3, host_threads=threads)
        s0 = g.stats()
        g.prefetch(2 if threads == 1 else 16)
        s = g.stats()
        fed = s["bits_bytes_fed"] - s0["bits_bytes_fed"]
        sec = s["feed_seconds"] - s0["feed_seconds"]
        res[f"gg_host_{threads}_threads"] = {"labels_per_s": fed / 8 / sec, "bytes": fed,
                                             "threads": threads}
        g.close()
    # the hybrid with the host generator as FEED: GPU numbers per second end to end
    g = Generator(walkers=W, seed=0x5EED0006, bit_source=3, host_threads=cores)
    o = torch.empty(W * 16, dtype=torch.int64, device="cuda")
    g.fill(o[: W])  # warm
    torch.cuda.synchronize()
    t = time.perf_counter()
    g.fill(o)
    torch.cuda.synchronize()
    dt = time.perf_counter() - t
    res["gpu_fill_fed_by_host_generator"] = {"numbers_per_s": o.numel() / dt,
                                             "labels": o.numel(), "walkers": W}
    g.close()
    res["host"] = {"nproc": cores}
    out = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "fig6.json")
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res))


if __name__ == "__main__":
    main()

"""Measure the GPU box (tool; SURVEY §7 step 0 "Measure the box first").

    nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/int_peak tools/int_peak.cu
    python tools/measure_box.py [out.json]

Records what the rooflines of DESIGN.md §6 rest on and MEASURED_PEAKS.json
lacks: the integer lane-op rate of the ALU pipe (LOP3), the FMA-heavy pipe
(IMAD) and both interleaved 1:1 (tools/int_peak.cu); HBM store-only and
copy GB/s; pinned H2D / D2H / bidirectional GB/s; host cores and the seed-bit
FEED rate (SplitMix64 counter hash into pinned chunks) on one core and on all.
"""
import json
import os
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402


def ev_time(fn, reps=5):
    best = 1e30
    for _ in range(reps):
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        best = min(best, a.elapsed_time(b) / 1e3)
    return best


def main():
    res = {}
    exe = os.path.join(ROOT, "tools", "int_peak")
    if not os.path.exists(exe):
        subprocess.run(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-o", exe,
                        exe + ".cu"], check=False)
    if os.path.exists(exe):
        out = subprocess.run([exe], capture_output=True, text=True, timeout=300)
        res["int_issue"] = json.loads(out.stdout.strip().splitlines()[-1])
    p = torch.cuda.get_device_properties(0)
    res["gpu"] = {"name": p.name, "sms": p.multi_processor_count,
                  "hbm_gib": p.total_memory / 2**30}
    try:
        import pynvml
        pynvml.nvmlInit()
        h = pynvml.nvmlDeviceGetHandleByIndex(0)
        res["gpu"]["sm_max_mhz"] = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
        res["gpu"]["mem_max_mhz"] = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_MEM)
    except Exception as e:  # noqa: BLE001
        res["gpu"]["nvml"] = str(e)

    n = 8 << 30
    x = torch.empty(n, dtype=torch.uint8, device="cuda")
    y = torch.empty(n, dtype=torch.uint8, device="cuda")
    res["hbm_store_gbs"] = n / ev_time(lambda: x.fill_(7)) / 1e9
    res["hbm_copy_gbs"] = 2 * n / ev_time(lambda: y.copy_(x)) / 1e9  # read + write
    del x, y
    torch.cuda.empty_cache()

    m = 1 << 30
    hbuf = torch.empty(m, dtype=torch.uint8).pin_memory()
    hbuf2 = torch.empty(m, dtype=torch.uint8).pin_memory()
    d = torch.empty(m, dtype=torch.uint8, device="cuda")
    d2 = torch.empty(m, dtype=torch.uint8, device="cuda")
    res["h2d_pinned_gbs"] = m / ev_time(lambda: d.copy_(hbuf, non_blocking=True)) / 1e9
    res["d2h_pinned_gbs"] = m / ev_time(lambda: hbuf.copy_(d, non_blocking=True)) / 1e9
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def both():
        cur = torch.cuda.current_stream()
        s1.wait_stream(cur)
        s2.wait_stream(cur)
        with torch.cuda.stream(s1):
            d.copy_(hbuf, non_blocking=True)
        with torch.cuda.stream(s2):
            hbuf2.copy_(d2, non_blocking=True)
        cur.wait_stream(s1)
        cur.wait_stream(s2)
    res["h2d_plus_d2h_gbs"] = 2 * m / ev_time(both) / 1e9

    res["host"] = {"nproc": os.cpu_count()}
    try:
        with open("/proc/cpuinfo") as f:
            res["host"]["cpu_model"] = next(ln.split(":", 1)[1].strip() for ln in f
                                            if ln.startswith("model name"))
    except (OSError, StopIteration):
        pass
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    for threads in (1, os.cpu_count() or 1):
        g = Generator(walkers=1 << 20, seed=1, host_threads=threads)
        s0 = g.stats()
        t = time.perf_counter()
        g.prefetch(64 if threads > 1 else 8)
        wall = time.perf_counter() - t
        s = g.stats()
        fed = s["bits_bytes_fed"] - s0["bits_bytes_fed"]
        res["host"][f"feed_{threads}_threads"] = {
            "gen_gbs": fed / (s["feed_seconds"] - s0["feed_seconds"]) / 1e9,
            "prefetch_gbs": fed / wall / 1e9, "bytes": fed}
        g.close()
    path = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "measured_box.json")
    with open(path, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res))


if __name__ == "__main__":
    main()

#!/usr/bin/env python
"""Benchmark of the B200 expander-walk PRNG (BASELINE.json metric, config C2).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...        (one rank per GPU)

A step = one bulk prng_fill of 2^30 uint32 numbers (= 2^29 64-bit labels,
the paper's numbers) from 2^20 walkers on the full-size expander (m = 2^32,
n = 2^65, l = l0 = 64) per GPU: Alg.2 x 512 draws per walker with the seed
bits resident in HBM (prefetched by the host FEED before the timed region).
Between steps the generator is rewound to the same checkpoint, so every step
walks the same 12 GiB of bits (larger than L2: no flush needed) and writes
4 GiB of labels.  Multi-GPU: walkers shard by rank with disjoint streams
(weak scaling, no collective on the data path); time = max over ranks.

`e2e` is the same metric through prng_fill_host with host buffers: host FEED
threads generate every bit, H2D copies, the walk, D2H of all numbers.
`--impl reference` times the CPU oracle (the paper's method as plain C) on
the host cores instead.

`--workload c5` runs config C5 instead (BJ:configs "2^34 numbers sharded over
1/2/4/8 B200"): 2^34 labels in total from 2^23 walkers split over
the ranks (strong scaling), each rank filling a reused 2 GiB buffer; value =
labels / summed fill time with each fill's bits prefetched (K-mode), e2e =
the same job with the host FEED streaming the bits during the walk (E-mode).
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

METRIC = "GNumbers/s (bulk fill and on-demand) per B200 and at 2/4/8 GPUs; % roofline"
UNIT = "GNumbers/s"
M32 = 1 << 32
SEED = 0x5EED0002
W_PER_GPU = 1 << 20
U32_PER_STEP = 1 << 30
LABELS_PER_STEP = U32_PER_STEP // 2          # 2^29 labels per GPU per step
DRAWS_PER_STEP = LABELS_PER_STEP // W_PER_GPU  # 512
BITS_BYTES_PER_LABEL = 24                     # 64 steps x 3 bits
# Algorithmic integer work per number ("64 neighbour evaluations,
# each ~4-6 integer ops minimum").  The fill kernel composes 4 steps into one
# affine map and issues ~311 SASS per number, fewer than 6 per step, so the
# roofline uses the survey's lower bound, 4 ops per step; the
# 6-op figure is reported beside it.
OPS_PER_STEP = 4
OPS_PER_LABEL = 64 * OPS_PER_STEP + 1         # + the emit
OPS_PER_LABEL_6 = 64 * 6 + 1
FILL_KERNEL = "gg_fill64t_tma_kernel"
WORKLOAD = ("C2 bulk prng_fill: m=2^32 (n=2^65), degree 7, l=l0=64, 2^20 walkers per GPU, "
            "2^30 uint32 numbers (2^29 64-bit labels) per GPU per step")


# --------------------------------------------------------------- CPU oracle
def _oracle_worker(args):
    t0, nwalkers, ndraws = args
    import oracle as O
    lib = O.lib()
    import numpy as np
    out = np.empty(ndraws, dtype=np.uint64)
    acc = 0
    for t in range(t0, t0 + nwalkers):
        lib.or_walker_draws(M32, 64, 64, SEED, t, 0, ndraws, out.ctypes.data)
        acc ^= int(out[-1])
    return acc


def oracle_rate(cores: int, walkers_per_core: int, draws: int):
    """Labels/s of `cores` single-threaded oracle processes on disjoint walkers."""
    import multiprocessing as mp
    ctx = mp.get_context("spawn")
    with ctx.Pool(cores) as pool:
        pool.map(_oracle_worker, [(0, 1, 1)] * cores)  # warm (load + build the .so)
        jobs = [(c * walkers_per_core * 1021 % (W_PER_GPU - walkers_per_core), walkers_per_core,
                 draws) for c in range(cores)]
        t = time.perf_counter()
        pool.map(_oracle_worker, jobs)
        dt = time.perf_counter() - t
    labels = cores * walkers_per_core * draws
    return labels / dt, labels, dt


def cpu_baseline_block(target_seconds: float = 8.0):
    cores = os.cpu_count() or 1
    # calibrate on one core, then size the sample to ~target_seconds wall
    r1, _, _ = oracle_rate(1, 64, 64)
    per_core = max(64 * 16, int(r1 * target_seconds))
    # the plain oracle on one core, then on all cores
    r1, l1, t1 = oracle_rate(1, max(1, int(r1 * 2.0) // 64), 64)
    draws = 64
    walkers = max(1, per_core // draws)
    rate, labels, dt = oracle_rate(cores, walkers, draws)
    return {
        "value": rate / 1e9, "unit": UNIT, "cores": cores, "kind": "oracle",
        "value_1core": r1 / 1e9, "sample_1core": f"{l1} labels on one core, {t1:.1f} s",
        "sample": (f"{labels} labels of the C2 workload (m=2^32, l=l0=64, seed 0x5EED0002): "
                   f"{cores} single-threaded oracle processes x {walkers} walkers x draws 0..{draws-1} "
                   f"(Alg.1 burn-in included), {dt:.1f} s wall"),
    }


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """SM clock and throttle reasons sampled during the run by two independent
    samplers: NVML in a thread (~2 ms; power every 8th sample) and
    `nvidia-smi -lms 20` in a subprocess (the recipe's clocks line).  Each
    NVML query is tried on its own, so one unsupported call does not stop the
    sampling.  start before the warm-up, mark(True/False) around the timed
    region: summary() keeps the samples taken inside it (NVML's if it has
    any, else nvidia-smi's), falling back to every sample under load if the
    region is shorter than the sampling period."""
    REASONS = (("hw_slowdown", 0x8), ("hw_thermal_slowdown", 0x40), ("sw_thermal_slowdown", 0x20),
               ("sw_power_cap", 0x4), ("hw_power_brake_slowdown", 0x80))

    def __init__(self, gpu_id: str, index: int = 0):
        self.gpu_id, self.index = gpu_id, index
        self.rows = {"nvml": [], "nvidia-smi": []}  # (t, sm_mhz, max_mhz, power_w, reasons)
        self.t0 = self.t1 = None
        self.stop = threading.Event()
        self.threads = []
        self.proc = None

    def __enter__(self):
        self._nvml()
        self._smi()
        return self

    def _nvml(self):
        try:
            import pynvml
            pynvml.nvmlInit()
            try:
                h = pynvml.nvmlDeviceGetHandleByUUID(self.gpu_id)
            except Exception:
                h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
        except Exception:
            return
        reasons_fn = getattr(pynvml, "nvmlDeviceGetCurrentClocksEventReasons", None) or \
            getattr(pynvml, "nvmlDeviceGetCurrentClocksThrottleReasons", None)

        def q(fn, *a):
            try:
                return fn(h, *a)
            except Exception:
                return None

        def run():
            mx = q(pynvml.nvmlDeviceGetMaxClockInfo, pynvml.NVML_CLOCK_SM)
            pw, i = 0.0, 0
            while not self.stop.is_set():
                if i % 8 == 0:
                    v = q(pynvml.nvmlDeviceGetPowerUsage)
                    pw = v / 1000.0 if v is not None else pw
                i += 1
                sm = q(pynvml.nvmlDeviceGetClockInfo, pynvml.NVML_CLOCK_SM)
                rs = q(reasons_fn) if reasons_fn else None
                if sm is not None and rs is not None:
                    self.rows["nvml"].append((time.perf_counter(), float(sm),
                                              float(mx if mx is not None else sm), pw, int(rs)))
                time.sleep(0.002)
        th = threading.Thread(target=run, daemon=True)
        th.start()
        self.threads.append(th)

    def _smi(self):
        fields = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
                  "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
                  "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", self.gpu_id, f"--query-gpu={fields}",
                 "--format=csv,noheader,nounits", "-lms", "20"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.proc = None
            return
        bits = (0x8, 0x40, 0x20, 0x4)

        def run():
            for line in self.proc.stdout:
                p = [x.strip() for x in line.split(",")]
                if len(p) == 7:
                    try:
                        rs = sum(b for b, v in zip(bits, p[3:]) if v == "Active")
                        self.rows["nvidia-smi"].append((time.perf_counter(), float(p[0]),
                                                        float(p[1]), float(p[2]), rs))
                    except ValueError:
                        pass
        th = threading.Thread(target=run, daemon=True)
        th.start()
        self.threads.append(th)

    def mark(self, start: bool):
        if start:
            self.t0 = time.perf_counter()
        else:
            self.t1 = time.perf_counter()

    def __exit__(self, *exc):
        self.stop.set()
        if self.proc is not None:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()
        for th in self.threads:
            th.join(timeout=1)

    def summary(self):
        def inside(rows):
            return [r for r in rows if self.t0 is not None and self.t1 is not None
                    and self.t0 <= r[0] <= self.t1]
        src, use, ins = None, [], []
        for name in ("nvml", "nvidia-smi"):
            rows = list(self.rows[name])
            ins = inside(rows)
            if len(ins) >= 3:
                src, use = name, ins
                break
        if not use:
            for name in ("nvml", "nvidia-smi"):
                rows = list(self.rows[name])
                if rows:
                    src, use, ins = name, rows, inside(rows)
                    break
        if not use:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unavailable"], "samples": 0}
        reasons = sorted({n for r in use for n, b in self.REASONS if r[4] & b})
        return {"sm_mhz": statistics.median(r[1] for r in use),
                "sm_max_mhz": max(r[2] for r in use), "reasons": reasons,
                "power_w_max": max(r[3] for r in use), "samples": len(use),
                "samples_in_timed_region": len(ins),
                "window": "timed region" if use is ins else "whole K-mode section (region < 3 samples)",
                "source": src,
                "samples_by_source": {k: len(v) for k, v in self.rows.items()}}


def committed_traffic():
    """dram read+write bytes per launch of the fill kernel from the committed
    ncu --set full capture of the default kernel, or None."""
    path = os.path.join("profiles", "r02_fill_table_ncu.json")
    try:
        with open(os.path.join(ROOT, path)) as f:
            d = json.load(f)
        gb = d["dram__bytes_read.sum"]["value"] + d["dram__bytes_write.sum"]["value"]
        return {"bytes": gb * 1e9, "source": f"{path} (ncu --set full, one launch)",
                "kernel": d.get("Kernel Name", {}).get("value")}
    except (OSError, KeyError, ValueError):
        return None


def sass_per_label():
    """Static SASS count per number of the fill kernel's interior draw
    (tools/sass_hist.py -> profiles/r02_fill_table_sass.txt), or None."""
    try:
        with open(os.path.join(ROOT, "profiles", "r02_fill_table_sass.txt")) as f:
            head = f.readline()
        return float(head.split("=")[1].split("per label")[0])
    except (OSError, IndexError, ValueError):
        return None


def measured_int_peak():
    """Interleaved LOP3/IMAD lane-op rate measured by tools/int_peak.cu on this
    pool's B200 (profiles/r01_measured_box.json), T ops/s, or None."""
    try:
        with open(os.path.join(ROOT, "profiles", "r01_measured_box.json")) as f:
            return float(json.load(f)["int_issue"]["lop3_imad_1to1_tops"])
    except (OSError, KeyError, ValueError):
        return None


def pcie_bound(h2d_bytes: float, d2h_bytes: float, labels: float):
    """Upper bound on e2e labels/s from the measured PCIe rates of this pool's
    box (profiles/r01_measured_box.json): the D2H bytes share the link with
    as many H2D bytes at the bidirectional rate, the rest of the H2D bytes
    run at the one-way rate."""
    try:
        with open(os.path.join(ROOT, "profiles", "r01_measured_box.json")) as f:
            mb = json.load(f)
        h2d, bi = float(mb["h2d_pinned_gbs"]) * 1e9, float(mb["h2d_plus_d2h_gbs"]) * 1e9
    except (OSError, KeyError, ValueError):
        return None
    both = min(h2d_bytes, d2h_bytes)
    t = 2 * both / bi + (h2d_bytes - both) / h2d + (d2h_bytes - both) / h2d
    return {"kind": "pcie", "h2d_gbs": h2d / 1e9, "bidir_gbs": bi / 1e9,
            "max_value": labels / t / 1e9, "source": "profiles/r01_measured_box.json"}


def _measured_h2d_gbs():
    try:
        with open(os.path.join(ROOT, "profiles", "r01_measured_box.json")) as f:
            return float(json.load(f)["h2d_pinned_gbs"])
    except (OSError, KeyError, ValueError):
        return None


def measured_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)
    except OSError:
        return {}


# ------------------------------------------------------------- our arm
def run_ours(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_banerjeebk12_b200 import Generator

    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    props = torch.cuda.get_device_properties(dev)
    stream = torch.cuda.current_stream()
    # the ranks of one node share the host cores for their FEED threads
    feed_threads = _feed_threads(world)

    def barrier():
        if world > 1:
            dist.barrier()

    def max_over_ranks(v: float) -> float:
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def per_rank(v: float) -> list:
        if world == 1:
            return [v]
        t = torch.zeros(world, dtype=torch.float64, device=dev)
        t[rank] = v
        dist.all_reduce(t)  # each slot is non-zero on exactly one rank
        return [float(x) for x in t.tolist()]

    # ---- K-mode: bits resident in HBM, one prng_fill per step
    g = Generator(walkers=W_PER_GPU, seed=SEED, walker_base=rank * W_PER_GPU, device=local_rank,
                  host_threads=feed_threads)
    g.prefetch(DRAWS_PER_STEP)
    g.mark()
    out = torch.empty(U32_PER_STEP, dtype=torch.int32, device=dev)
    gpu_id = getattr(props, "uuid", None)
    gpu_id = f"GPU-{gpu_id}" if gpu_id is not None else str(local_rank)
    clk = ClockSampler(gpu_id, local_rank).__enter__()  # running before the warm-up
    for _ in range(args.warmup):
        g.rewind()
        g.fill(out)
    torch.cuda.synchronize()
    ev0 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    ev1 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    start, end = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    launches0 = g.stats()["kernel_launches"]
    barrier()
    torch.cuda.synchronize()
    clk.mark(True)
    start.record(stream)
    for i in range(args.steps):
        g.rewind()
        ev0[i].record(stream)
        g.fill(out)
        ev1[i].record(stream)
    end.record(stream)
    torch.cuda.synchronize()
    clk.mark(False)
    clk.__exit__(None, None, None)
    barrier()
    launches = g.stats()["kernel_launches"] - launches0
    ms_ranks = per_rank(start.elapsed_time(end))
    ms = max(ms_ranks)
    step_ms = [a.elapsed_time(b) for a, b in zip(ev0, ev1)]
    kern_ms = statistics.mean(step_ms)
    labels_total = world * LABELS_PER_STEP * args.steps
    value = labels_total / (ms / 1e3) / 1e9

    peaks = measured_peaks()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    peak_ops = props.multi_processor_count * 128 * sm_max * 1e6  # int lanes/clk/SM x clock
    achieved_ops = LABELS_PER_STEP * OPS_PER_LABEL / (kern_ms / 1e3)
    tr = committed_traffic()
    roofline = {
        "bound": "alu", "achieved": achieved_ops / 1e12, "peak": peak_ops / 1e12,
        "unit": "Tops/s (32-bit integer ops)", "frac": achieved_ops / peak_ops,
        "traffic": tr["bytes"] if tr else None,
        "traffic_note": (f"DRAM bytes per launch, {tr['source']}; algorithmic bytes per launch "
                         f"{LABELS_PER_STEP * (BITS_BYTES_PER_LABEL + 8):.4g}") if tr else None,
        "kernel": FILL_KERNEL,
        "kernel_ms": kern_ms, "ops_per_label": OPS_PER_LABEL,
        "kernel_ms_median_min_max": [statistics.median(step_ms), min(step_ms), max(step_ms)],
        "peak_basis": (f"{props.multi_processor_count} SMs x 128 int lanes/clk (ALU 64 + FMA 64, "
                       f"issue 4x32) x {sm_max:.0f} MHz (MEASURED_PEAKS sm_max_mhz)"),
        "peak_measured": measured_int_peak(),
        "peak_measured_note": ("tools/int_peak.cu, LOP3/IMAD interleaved 1:1 "
                               "(profiles/r01_measured_box.json); frac uses the derived peak"),
        "hbm_gbs_achieved": LABELS_PER_STEP * (BITS_BYTES_PER_LABEL + 8) / (kern_ms / 1e3) / 1e9,
        "hbm_gbs_peak": peaks.get("hbm_gbs"),
        # the same time against SURVEY §8(d)'s 6-op step (above 1: composing
        # 4 steps into one affine map needs fewer than 6 instructions per step)
        "frac_at_6_ops_per_step": (LABELS_PER_STEP * OPS_PER_LABEL_6 / (kern_ms / 1e3)) / peak_ops,
    }
    spl = sass_per_label()
    if spl:
        # the kernel's own instruction stream against the issue peak (one warp
        # instruction per SMSP per cycle = the same 128 lanes/clk/SM)
        roofline["executed_sass_per_label"] = spl
        roofline["executed_frac"] = LABELS_PER_STEP * spl / (kern_ms / 1e3) / peak_ops
        roofline["executed_note"] = ("static SASS of the interior draw (profiles/r02_fill_table_sass.txt) "
                                     "x labels / kernel time / peak")
    # (no oracle call here: the task reserves oracle/ for the cpu_baseline leg;
    # parity of this exact launch configuration is tests/test_gpu_generator.py's
    # full-size sampled check)
    res = {"value": value, "ms": ms, "roofline": roofline, "clocks": clk.summary(),
           "launches": launches, "kern_ms": kern_ms,
           "per_rank": [{"rank": r, "ms": x, "value": LABELS_PER_STEP * args.steps / (x / 1e3) / 1e9}
                        for r, x in enumerate(ms_ranks)]}
    g.close()
    del out
    torch.cuda.empty_cache()

    # ---- f1: l = 1 ("emit every vertex"): 4 B read + 8 B written
    # per number, HBM-bound; 2^20 walkers x 1024 draws, bits resident
    if not args.no_l1:
        g = Generator(walkers=W_PER_GPU, seed=SEED, walk_len=1, walker_base=rank * W_PER_GPU,
                      device=local_rank, host_threads=feed_threads)
        D1 = 1024
        g.prefetch(D1)
        g.mark()
        o1 = torch.empty(W_PER_GPU * D1, dtype=torch.int64, device=dev)
        for _ in range(args.warmup):
            g.rewind()
            g.fill(o1)
        e0 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
        e1 = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
        torch.cuda.synchronize()
        for i in range(args.steps):
            g.rewind()
            e0[i].record(stream)
            g.fill(o1)
            e1[i].record(stream)
        torch.cuda.synchronize()
        ms1 = max_over_ranks(statistics.median(a.elapsed_time(b) for a, b in zip(e0, e1)))
        labels1 = W_PER_GPU * D1
        gbs = labels1 * 12 / (ms1 / 1e3) / 1e9
        res["l1_fill"] = {
            "config": "l = 1 (one 3-bit step per number), m = 2^32, 2^20 walkers x 1024 draws per GPU",
            "value": world * labels1 / (ms1 / 1e3) / 1e9, "unit": UNIT, "ms_kernel": ms1,
            "roofline": {"bound": "hbm", "achieved": gbs, "peak": measured_peaks().get("hbm_gbs"),
                         "unit": "GB/s", "frac": gbs / measured_peaks().get("hbm_gbs", 6460.9),
                         "bytes_per_number": 12, "kernel": "gg_fill_l1_tma_kernel"}}
        g.close()
        del o1
        torch.cuda.empty_cache()

    # ---- on-demand: every thread calls prng_next S = 100 times (Fig.4 batch)
    if not args.no_ondemand:
        S = 100
        g = Generator(walkers=W_PER_GPU, seed=SEED + 1, walker_base=rank * W_PER_GPU,
                      device=local_rank, host_threads=feed_threads)
        xo = torch.empty(W_PER_GPU, dtype=torch.int64, device=dev)
        g.epoch_begin(W_PER_GPU, S * (args.warmup + 1))
        for _ in range(args.warmup):
            g.consume(W_PER_GPU, uniform=S, xor_out=xo)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        a.record(stream)
        g.consume(W_PER_GPU, uniform=S, xor_out=xo)
        b.record(stream)
        torch.cuda.synchronize()
        g.epoch_end()
        od_ms = max_over_ranks(a.elapsed_time(b))
        res["on_demand"] = {"uniform_S100": world * W_PER_GPU * S / (od_ms / 1e3) / 1e9,
                            "unit": UNIT, "draws": world * W_PER_GPU * S, "ms": od_ms,
                            "what": "gg_consume: 2^20 threads/GPU x 100 prng_next each, bits resident",
                            "roofline_frac_uniform": (W_PER_GPU * S * OPS_PER_LABEL / (od_ms / 1e3))
                            / (props.multi_processor_count * 128 * sm_max * 1e6)}
        g.close()
        torch.cuda.empty_cache()
        res["on_demand"].update(ondemand_shaped(rank, world, local_rank, stream, max_over_ranks))
        torch.cuda.empty_cache()

    # ---- on-demand consumers of the paper at full size (C3, C4), one run each
    if not args.no_apps:
        res["apps"] = run_apps(args, rank, world, local_rank, max_over_ranks, feed_threads)
        torch.cuda.empty_cache()

    # ---- e2e: host buffers through prng_fill_host (FEED + H2D + walk + D2H)
    if not args.no_e2e:
        e2e_steps = max(1, min(args.steps, args.e2e_steps))
        g = Generator(walkers=W_PER_GPU, seed=SEED, walker_base=rank * W_PER_GPU,
                      device=local_rank, epoch_draws=int(os.environ.get("GG_E2E_D", "16")),
                      host_threads=feed_threads)
        host = torch.empty(U32_PER_STEP, dtype=torch.int32).pin_memory()
        g.fill_host(host, n=W_PER_GPU * 2 * 16)  # warm (allocations, feed threads)
        g.mark()
        s0 = g.stats()
        barrier()
        torch.cuda.synchronize()
        t = time.perf_counter()
        for _ in range(e2e_steps):
            g.rewind()
            g.fill_host(host)
        torch.cuda.synchronize()
        dt_ranks = per_rank(time.perf_counter() - t)
        dt = max(dt_ranks)
        s1 = g.stats()
        res["e2e"] = {
            "per_rank": [LABELS_PER_STEP * e2e_steps / x / 1e9 for x in dt_ranks],
            "value": world * LABELS_PER_STEP * e2e_steps / dt / 1e9, "unit": UNIT,
            "h2d_bytes_per_step": (s1["h2d_bytes"] - s0["h2d_bytes"]) // e2e_steps,
            "d2h_bytes_per_step": (s1["d2h_bytes"] - s0["d2h_bytes"]) // e2e_steps,
            "steps": e2e_steps,
            "feed_s_per_step": (s1["feed_seconds"] - s0["feed_seconds"]) / e2e_steps,
            "api": "prng_fill_host (host FEED threads -> pinned -> H2D -> walk -> D2H to pinned)",
            "host_threads": feed_threads,
            "feed_pace_mbs": s1["feed_pace_mbs"],
        }
        b = pcie_bound(res["e2e"]["h2d_bytes_per_step"], res["e2e"]["d2h_bytes_per_step"],
                       LABELS_PER_STEP)
        if b:
            b["frac"] = res["e2e"]["value"] / world / b["max_value"]
            res["e2e"]["bound"] = b
        g.close()
    return res


# ------------------------------------------------------- C5 scaling sweep
C5_LABELS = 1 << 34          # BJ:configs "2^34 numbers sharded over 1/2/4/8 B200"
C5_WALKERS = 1 << 23         # W = 2^23 in total, split G ways (strong scaling)
C5_CHUNK = 1 << 28           # labels per fill: a 2 GiB reused u64 buffer per GPU
C5_SEED = 0x5EED0005
C5_WORKLOAD = ("C5 scaling sweep: 2^34 64-bit labels in total (m=2^32, l=l0=64), 2^23 walkers "
               "split over the GPUs (global walker ids, disjoint seed-bit streams), each GPU "
               "filling a reused 2 GiB buffer (2^28 labels per prng_fill)")


def run_c5(args, rank, world, local_rank):
    """One step = the whole C5 job.  K-mode (value): per chunk the chunk's bits
    are made resident by prng_prefetch (host FEED + H2D, untimed), then the
    fill is timed with CUDA events; time = max over ranks of the summed fill
    times.  E-mode (e2e): a second generator on the same seed runs the same
    job through prng_fill with the host FEED and H2D overlapped with the
    walk (the paper's regime), wall time between device synchronisations,
    max over ranks; the last label is read back to the host."""
    import torch
    import torch.distributed as dist
    from paper_conf_ipps_banerjeebk12_b200 import Generator

    if C5_WALKERS % world or (C5_LABELS // world) % C5_CHUNK:
        raise SystemExit(f"C5 needs world in (1, 2, 4, 8, ...); got {world}")
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    props = torch.cuda.get_device_properties(dev)
    stream = torch.cuda.current_stream()
    feed_threads = _feed_threads(world)
    Wr = C5_WALKERS // world
    base = rank * Wr
    Lr = C5_LABELS // world
    chunks = Lr // C5_CHUNK
    draws_per_chunk = C5_CHUNK // Wr

    def max_over_ranks(v: float) -> float:
        if world == 1:
            return v
        t = torch.tensor([v], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    def barrier():
        if world > 1:
            dist.barrier()

    out = torch.empty(C5_CHUNK, dtype=torch.int64, device=dev)
    gpu_id = getattr(props, "uuid", None)
    gpu_id = f"GPU-{gpu_id}" if gpu_id is not None else str(local_rank)
    clk = ClockSampler(gpu_id, local_rank).__enter__()

    def k_job(timed: bool):
        g = Generator(walkers=Wr, seed=C5_SEED, walker_base=base, device=local_rank,
                      host_threads=feed_threads)
        kms, launches = 0.0, 0
        for c in range(chunks):
            g.prefetch(draws_per_chunk)
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            l0 = g.stats()["kernel_launches"]
            a.record(stream)
            g.fill(out)
            b.record(stream)
            b.synchronize()
            launches += g.stats()["kernel_launches"] - l0
            kms += a.elapsed_time(b)
        g.close()
        return kms, launches

    # warm-up: one chunk's worth of work per warm-up step (allocations, feed threads, clocks)
    for _ in range(args.warmup):
        g = Generator(walkers=Wr, seed=C5_SEED, walker_base=base, device=local_rank,
                      host_threads=feed_threads)
        g.prefetch(draws_per_chunk)
        g.fill(out)
        g.close()
    torch.cuda.synchronize()
    barrier()
    clk.mark(True)
    k_ms, launches = [], 0
    for _ in range(args.steps):
        ms, n = k_job(True)
        k_ms.append(max_over_ranks(ms))
        launches += n
    clk.mark(False)
    clk.__exit__(None, None, None)
    ms = sum(k_ms)
    value = C5_LABELS * args.steps / (ms / 1e3) / 1e9
    peaks = measured_peaks()
    sm_max = float(peaks.get("sm_max_mhz", 1965.0))
    peak_ops = props.multi_processor_count * 128 * sm_max * 1e6
    per_fill_ms = statistics.mean(k_ms) / chunks
    achieved = C5_CHUNK * OPS_PER_LABEL / (per_fill_ms / 1e3)
    roofline = {
        "bound": "alu", "achieved": achieved / 1e12, "peak": peak_ops / 1e12,
        "unit": "Tops/s (32-bit integer ops)", "frac": achieved / peak_ops, "traffic": None,
        "kernel": FILL_KERNEL, "kernel_ms": per_fill_ms, "ops_per_label": OPS_PER_LABEL,
        "note": "per-launch time = summed fill time / fills (max over ranks)"}

    # E-mode: the same job with the bits streamed by the host FEED during the walk
    e2e = None
    if not args.no_e2e:
        g = Generator(walkers=Wr, seed=C5_SEED, walker_base=base, device=local_rank,
                      epoch_draws=16, host_threads=feed_threads)
        host_last = torch.empty(1, dtype=torch.int64).pin_memory()
        s0 = g.stats()
        barrier()
        torch.cuda.synchronize()
        t = time.perf_counter()
        for c in range(chunks):
            g.fill(out)
        host_last.copy_(out[-1:], non_blocking=False)
        torch.cuda.synchronize()
        dt = max_over_ranks(time.perf_counter() - t)
        s1 = g.stats()
        g.close()
        e2e = {"value": C5_LABELS / dt / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": s1["h2d_bytes"] - s0["h2d_bytes"],
               "d2h_bytes_per_step": 8, "steps": 1, "ms_wall": dt * 1e3,
               "feed_s": s1["feed_seconds"] - s0["feed_seconds"], "host_threads": feed_threads,
               "api": "prng_fill into the reused device buffer, host FEED -> pinned -> H2D "
                      "overlapped with the walk; last label read back"}
        b = pcie_bound(e2e["h2d_bytes_per_step"], 8, C5_LABELS / world)
        if b:
            b["frac"] = e2e["value"] / world / b["max_value"]
            e2e["bound"] = b
    return {"value": value, "ms": ms, "roofline": roofline, "clocks": clk.summary(),
            "launches": launches, "e2e": e2e, "walkers_per_gpu": Wr, "chunks_per_gpu": chunks,
            "draws_per_chunk": draws_per_chunk}


def host_info():
    """nproc and CPU model of the box (SURVEY §8(d) reporting rules)."""
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for ln in f:
                if ln.startswith("model name"):
                    model = ln.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"nproc": os.cpu_count(), "cpu_model": model}


def _feed_threads(world):
    """Host FEED threads per rank: the ranks of a node share its cores
    (GG_BENCH_FEED_THREADS overrides, for A/B runs)."""
    if os.environ.get("GG_BENCH_FEED_THREADS"):
        return int(os.environ["GG_BENCH_FEED_THREADS"])
    local_world = int(os.environ.get("LOCAL_WORLD_SIZE", str(world)))
    return max(1, (os.cpu_count() or 1) // max(1, local_world))


def _hash32(t, r):
    """Integer hash of (thread, round) on the device (activity pattern only)."""
    x = (t * 2654435761 + r * 0x27D4EB2F + 0x165667B1) & 0xFFFFFFFF
    x = ((x ^ (x >> 16)) * 0x45D9F3B) & 0xFFFFFFFF
    x = ((x ^ (x >> 16)) * 0x45D9F3B) & 0xFFFFFFFF
    return x ^ (x >> 16)


def ondemand_shaped(rank, world, local_rank, stream, max_over_ranks):
    """SURVEY §8(d) on-demand consumers shaped like the paper's workloads,
    bits resident (draws / sum of consumer-kernel time):
      lr_shaped: 2^24 threads over 24 rounds; thread t is active in round r
                 iff hash(t, r) < (7/8)^r * 2^32 and then makes one prng_next
                 (Alg.3's per-round draw with the FIS survival rate);
                 lr_shaped_compact: the same active counts as slots 0..A_r-1;
      mc_shaped: 2^20 threads, each a geometric number of draws with mean 200
                 (C4's draws per photon), capped at 600, diverging in warps."""
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    dev = torch.device("cuda", local_rank)
    out = {}
    # LR-shaped
    W, R = 1 << 24, 24
    # 2^24 walkers fill the 24-bit walker-id space (R9), so the ranks run this
    # replicated consumer (like list ranking's Phase I) on seeds of their own
    g = Generator(walkers=W, seed=SEED + 2 + 1000 * rank, device=local_rank,
                  host_threads=_feed_threads(world))
    t = torch.arange(W, dtype=torch.int64, device=dev)
    counts = []
    for r in range(R):
        thr = int((7 / 8) ** r * 2**32)
        counts.append((_hash32(t, r) < thr).to(torch.int32))
    draws = int(sum(int(c.sum().item()) for c in counts))
    g.epoch_begin(W, R)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
          for _ in range(R)]
    torch.cuda.synchronize()
    for r in range(R):
        ev[r][0].record(stream)
        g.consume(W, counts=counts[r])
        ev[r][1].record(stream)
    torch.cuda.synchronize()
    ms = max_over_ranks(sum(a.elapsed_time(b) for a, b in ev))
    out["lr_shaped"] = world * draws / (ms / 1e3) / 1e9
    out["lr_shaped_detail"] = {"threads": W, "rounds": R, "draws": world * draws, "ms": ms,
                               "launches": R, "counts_bytes_read": R * W * 4}
    # the same rounds with the active threads compacted to slots 0..A_r-1, as
    # gg_list_rank runs them (walker = active slot, reading R16')
    active = [int(c.sum().item()) for c in counts]
    g.epoch_end()
    g.close()
    del counts, t
    torch.cuda.empty_cache()
    # 2^24 walkers fill the 24-bit walker-id space (R9), so the ranks run this
    # replicated consumer (like list ranking's Phase I) on seeds of their own
    g = Generator(walkers=W, seed=SEED + 2 + 1000 * rank, device=local_rank,
                  host_threads=_feed_threads(world))
    g.epoch_begin(W, R)
    torch.cuda.synchronize()
    for r in range(R):
        ev[r][0].record(stream)
        g.consume(active[r], uniform=1)
        ev[r][1].record(stream)
    torch.cuda.synchronize()
    g.epoch_end()
    ms = max_over_ranks(sum(a.elapsed_time(b) for a, b in ev))
    out["lr_shaped_compact"] = world * draws / (ms / 1e3) / 1e9
    out["lr_shaped_compact_ms"] = ms
    g.close()
    torch.cuda.empty_cache()
    # MC-shaped
    W, mean, cap = 1 << 20, 200, 600
    gen = torch.Generator(device="cpu").manual_seed(0x5EED0004 + rank)
    u = torch.rand(W, generator=gen, dtype=torch.float64)
    c = torch.clamp(torch.ceil(torch.log1p(-u) / math.log1p(-1 / mean)), 1, cap).to(torch.int32)
    draws = int(c.sum().item())
    c = c.to(dev)
    g = Generator(walkers=W, seed=SEED + 3, walker_base=rank * W, device=local_rank,
                  host_threads=_feed_threads(world))
    g.epoch_begin(W, cap)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    a.record(stream)
    g.consume(W, counts=c)
    b.record(stream)
    torch.cuda.synchronize()
    g.epoch_end()
    ms = max_over_ranks(a.elapsed_time(b))
    out["mc_shaped"] = world * draws / (ms / 1e3) / 1e9
    out["mc_shaped_detail"] = {"threads": W, "mean": mean, "cap": cap, "draws": world * draws,
                               "ms": ms, "launches": 1}
    g.close()
    return out


def run_apps(args, rank, world, local_rank, max_over_ranks, feed_threads=0):
    """C3 list ranking (2^24 nodes, replica per GPU) and C4 Monte Carlo (2^20
    threads per GPU, 20 photons each, ~2^32 draws per GPU; integer tallies
    all-reduced over ranks).  Numbers are device-timed inside the C ABI."""
    import torch

    import inputs
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    dev = torch.device("cuda", local_rank)
    out = {}
    # C3: list ranking of a 2^24-node random list.  With world > 1 the ranks
    # share Phase II (sublist walks) and exchange the splitter records
    # (allgather) and reduced-list ranks (allreduce) over NCCL.
    from paper_conf_ipps_banerjeebk12_b200 import dist as gd_
    coll = gd_.Collective(device=dev) if world > 1 else None
    n = 1 << 24
    succ, pred, head = inputs.random_list(n, 0x5EED0003)
    g = Generator(walkers=n, seed=0x5EED0003, device=local_rank, host_threads=feed_threads)
    s_t, p_t = torch.from_numpy(succ).to(dev), torch.from_numpy(pred).to(dev)
    # one untimed call (scratch pool, feed threads), then the median of 3
    rank_t, info = g.list_rank(s_t, p_t, head, collective=coll)
    walls, infos = [], []
    for _ in range(3):
        del rank_t
        torch.cuda.synchronize()
        t = time.perf_counter()
        rank_t, info = g.list_rank(s_t, p_t, head, collective=coll)
        torch.cuda.synchronize()
        walls.append(max_over_ranks(time.perf_counter() - t))
        infos.append(info)
    order = sorted(range(3), key=lambda i: walls[i])
    wall, info = walls[order[1]], infos[order[1]]
    ok = int(rank_t[head].item()) == 0 and int(rank_t.max().item()) == n - 1
    dev_us = info["phase1_us"] + info["phase2_us"] + info["phase3_us"]
    out["list_ranking"] = {
        "config": "C3: random list of 2^24 nodes, walker = active slot, b(u) = bit 63",
        "splitter_exchange": world > 1,
        "rounds": info["rounds"], "reduced": info["reduced"], "splitters": info["splitters"],
        "draws": info["draws"], "ms_device": dev_us / 1e3, "ms_wall": wall * 1e3,
        "ms_wall_runs": [w * 1e3 for w in walls], "timing": "median of 3 after 1 untimed call",
        "phase_ms": [info["phase1_us"] / 1e3, info["phase2_us"] / 1e3, info["phase3_us"] / 1e3],
        "draws_per_s_e2e": info["draws"] / wall / 1e9, "unit": "GNumbers/s",
        "ranks_ok": ok, "feed_pace_mbs": g.stats()["feed_pace_mbs"],
        "note": "on-demand: the host feeds exactly the draws of each round after learning the "
                "active count (FEED + H2D inside the measured time)"}
    h2d = _measured_h2d_gbs()
    if h2d:
        floor = info["draws"] * BITS_BYTES_PER_LABEL / (h2d * 1e9)
        out["list_ranking"]["pcie_floor_ms"] = floor * 1e3
        out["list_ranking"]["frac_of_pcie_floor"] = floor / wall
    # the host FEED pipeline alone on the same windows: the per-round active
    # counts of this run replayed through prng_epoch_begin / prng_epoch_end
    # (bits generated by the feed threads into pinned chunks and copied,
    # no kernels) -- the rate this host can supply C3's bits at
    rr = torch.empty(n, dtype=torch.int32, device=dev)
    g.list_rank(s_t, p_t, head, removed_round=rr, collective=coll)
    gone = torch.bincount(rr[rr >= 0].long(), minlength=info["rounds"]).cpu().tolist()
    act = [n]
    for r in range(info["rounds"]):
        act.append(act[-1] - gone[r])   # act[r] = A_r; act[rounds] = Phase II's splitter draw
    g2 = Generator(walkers=n, seed=0x5EED0003, device=local_rank, host_threads=feed_threads)
    g2.epoch_reserve(n, 1)
    pipe = []
    for _ in range(2):
        torch.cuda.synchronize()
        t = time.perf_counter()
        for a in act:
            g2.epoch_begin(a, 1)
            g2.epoch_end()
        torch.cuda.synchronize()
        pipe.append(time.perf_counter() - t)
    g2.close()
    feed_ms = min(pipe) * 1e3
    out["list_ranking"]["feed_pipeline_ms"] = feed_ms
    out["list_ranking"]["feed_pipeline_gbs"] = sum(act) * BITS_BYTES_PER_LABEL / (feed_ms / 1e3) / 1e9
    out["list_ranking"]["frac_of_feed_pipeline"] = feed_ms / (wall * 1e3)
    g.close()
    del s_t, p_t, rank_t, rr
    torch.cuda.empty_cache()
    # C4: Monte Carlo photon migration, R19 slab
    from paper_conf_ipps_banerjeebk12_b200 import dist as gd
    thread0, T, T_total = gd.mc_shard(rank, world, W_PER_GPU)
    P_per = 20
    layers = ((1.37, 1.0, 100.0, 0.9, 0.1), (1.37, 1.0, 10.0, 0.0, 0.1), (1.37, 2.0, 10.0, 0.7, 0.2))
    # one untimed run on a throw-away handle (epoch windows, scratch pool, feed
    # threads' first touch: the first run of a process takes about twice as
    # long), then the median of 3 full runs, each on a fresh handle (the same
    # photons and draws every time)
    gw = Generator(walkers=T, seed=0x5EED0004, walker_base=thread0, device=local_rank,
                   host_threads=feed_threads)
    gw.mc_run(layers, photons_total=2 * T_total, threads=T, threads_total=T_total, thread0=thread0,
              epoch_draws=192)
    gw.close()
    runs = []
    for _ in range(3):
        g = Generator(walkers=T, seed=0x5EED0004, walker_base=thread0, device=local_rank,
                      host_threads=feed_threads)
        torch.cuda.synchronize()
        t = time.perf_counter()
        r = g.mc_run(layers, photons_total=P_per * T_total, threads=T, threads_total=T_total,
                     thread0=thread0, epoch_draws=192)
        runs.append((max_over_ranks(time.perf_counter() - t), r))
        if len(runs) < 3:
            g.close()
    runs_sorted = sorted(runs, key=lambda v: v[0])
    wall, r = runs_sorted[1]
    tal = gd.allreduce_tallies(r["tallies"], device=dev)  # exact int64 sums (NCCL over NVLink)
    draws = r["draws"] * world
    kern = max_over_ranks(r["kernel_us"] / 1e6)
    out["monte_carlo"] = {
        "config": "C4: R19 3-layer slab, 2^20 threads/GPU x 20 photons, 3 draws per iteration",
        "photons": P_per * T * world, "draws": draws, "epochs": r["epochs"],
        "draws_per_s_kernel": draws / kern / 1e9, "draws_per_s_e2e": draws / wall / 1e9,
        "unit": "GNumbers/s", "ms_wall": wall * 1e3, "ms_kernel": kern * 1e3,
        "ms_wall_runs": [w * 1e3 for w, _ in runs], "timing": "median of 3 after 1 untimed run",
        "R_d": tal[2] / tal[0], "T_t": tal[3] / tal[0], "specular": tal[1] / tal[0],
        "absorbed": [v / tal[0] for v in tal[5:]], "conserved": tal[0] == sum(tal[1:]),
        "host_bits_GB_used": draws * BITS_BYTES_PER_LABEL / 1e9,
        "host_bits_GB_fed": r["walker_epochs_fed"] * 192 * BITS_BYTES_PER_LABEL / 1e9 * world}
    if h2d:  # per rank: its own fed bytes over its own link
        floor = r["walker_epochs_fed"] * 192 * BITS_BYTES_PER_LABEL / (h2d * 1e9)
        out["monte_carlo"]["pcie_floor_ms"] = floor * 1e3
        out["monte_carlo"]["frac_of_pcie_floor"] = floor / wall
    g.close()
    return out


def _free_port() -> int:
    import socket
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def self_launch(n: int) -> int:
    """`bench.py --gpus N` run without a launcher: re-exec this script as N
    ranks through torch.distributed.run (one process per GPU, rendezvous on
    127.0.0.1).  The children see WORLD_SIZE, so they never spawn again.
    NCCL's INIT log (communicator size per rank) goes to stderr; the ranks'
    stdout is forwarded line by line, so the one JSON line rank 0 prints is
    the only line this process writes to stdout."""
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    env["GG_BENCH_SELF_LAUNCHED"] = "1"
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}",
           os.path.abspath(__file__)] + sys.argv[1:]
    p = subprocess.Popen(cmd, env=env, stdout=subprocess.PIPE, text=True)
    for line in p.stdout:
        if line.lstrip().startswith("{"):
            sys.stdout.write(line)
            sys.stdout.flush()
        else:
            sys.stderr.write(line)
    return p.wait()


def numa_nodes() -> int:
    try:
        return sum(1 for d in os.listdir("/sys/devices/system/node")
                   if d.startswith("node") and d[4:].isdigit())
    except OSError:
        return 1


def launch_probe(args, rank, world):
    """--launch-probe: the multi-rank plumbing of the bench without a GPU
    (process group, barrier, max over ranks, per-rank gather, one JSON line
    from rank 0).  Run by tests/test_bench_launch.py with gloo on CPU."""
    import torch
    import torch.distributed as dist
    if world > 1:
        dist.barrier()
        t = torch.tensor([float(rank + 1)], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        mx = float(t.item())
        per = [None] * world
        dist.all_gather_object(per, {"rank": rank, "value": float(rank + 1)})
    else:
        mx, per = 1.0, [{"rank": 0, "value": 1.0}]
    if rank == 0:
        print(json.dumps({"metric": METRIC, "launch_probe": True, "n_gpus": world,
                          "gpus_requested": args.gpus, "max_over_ranks": mx, "per_rank": per,
                          "backend": dist.get_backend() if world > 1 else None,
                          "feed_threads_per_rank": _feed_threads(world)}))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--launch-probe", action="store_true",
                    help="plumbing check only: process group + one JSON line, no GPU work")
    ap.add_argument("--steps", type=int, default=None, help="default 10 (C2), 1 (C5)")
    ap.add_argument("--workload", default="c2", choices=["c2", "c5"],
                    help="c2: bulk fill per GPU (weak scaling, default); c5: 2^34 labels split "
                         "over the GPUs (strong scaling)")
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-ondemand", action="store_true")
    ap.add_argument("--no-apps", action="store_true")
    ap.add_argument("--no-l1", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=8.0)
    args = ap.parse_args()
    if args.steps is None:
        args.steps = 1 if args.workload == "c5" else 10
    if args.warmup < 3:
        args.warmup = 3

    if args.gpus < 1:
        raise SystemExit("--gpus must be >= 1")
    if args.impl == "reference":
        # the oracle on the host cores: rank 0 alone (or the single process)
        if int(os.environ.get("RANK", "0")) != 0:
            return 0
        return run_reference(args, int(os.environ.get("WORLD_SIZE", str(args.gpus))))
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        return self_launch(args.gpus)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        raise SystemExit(f"bench.py: --gpus {args.gpus} but the launcher started {world} ranks")
    # test hooks: run the multi-rank path on one GPU (gloo, shared device)
    backend = os.environ.get("GG_DIST_BACKEND", "gloo" if args.launch_probe else "nccl")
    if "GG_FORCE_DEVICE" in os.environ:
        local_rank = int(os.environ["GG_FORCE_DEVICE"])
    if world > 1:
        # communicator size per rank in NCCL's INIT log (a self-launched run
        # forwards these non-JSON lines to stderr)
        os.environ.setdefault("NCCL_DEBUG", "INFO")
        os.environ.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
        # multi-socket hosts: each rank's FEED threads on its GPU's NUMA-local cores
        if numa_nodes() > 1:
            os.environ.setdefault("GG_FEED_PIN", "1")

    if args.launch_probe:
        if world > 1:
            import torch.distributed as dist
            dist.init_process_group(backend)
        launch_probe(args, rank, world)
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()
        return 0

    # CPU baseline first (spawned processes; before CUDA is initialised)
    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline_block(args.cpu_seconds)

    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        else:
            dist.init_process_group(backend)
    if args.workload == "c5":
        res = run_c5(args, rank, world, local_rank)
        if rank == 0:
            print(json.dumps({
                "metric": METRIC, "value": res["value"], "unit": UNIT, "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["ms"] / args.steps,
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "u64",
                "data": "synthetic (SplitMix64 counter-hash seed bits, reading R9)",
                "config": {"workload": C5_WORKLOAD, "number": "one 64-bit vertex label",
                           "walkers_per_gpu": res["walkers_per_gpu"],
                           "fills_per_gpu_per_step": res["chunks_per_gpu"],
                           "draws_per_fill": res["draws_per_chunk"],
                           "bits": "each fill's bits made resident by prng_prefetch (untimed); "
                                   "value = labels / summed fill kernel time (K-mode)",
                           "l2": "inputs larger than L2 (>= 6 GiB of bits per fill)",
                           "parallelism": f"walker shards dp{world}, no data-path collective"},
                "roofline": res["roofline"], "cpu_baseline": cpu, "e2e": res["e2e"],
                "clocks": res["clocks"], "gpu_launches": res["launches"], "host": host_info()}))
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()
        return 0
    res = run_ours(args, rank, world, local_rank)
    if rank == 0:
        line = {
            "metric": METRIC, "value": res["value"], "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["ms"] / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic (SplitMix64 counter-hash seed bits, reading R9)",
            "config": {"workload": WORKLOAD, "number": "one 64-bit vertex label (the paper's unit)",
                       "u32_numbers_per_s": 2 * res["value"] * 1e9,
                       "walkers_per_gpu": W_PER_GPU, "labels_per_gpu_per_step": LABELS_PER_STEP,
                       "bits": "resident in HBM (prng_prefetch before timing), rewound each step",
                       "l2": "inputs larger than L2 (12 GiB of bits read per GPU per step)",
                       "parallelism": f"walker shards dp{world}, no data-path collective"},
            "roofline": res["roofline"], "cpu_baseline": cpu, "e2e": res.get("e2e"),
            "clocks": res["clocks"], "gpu_launches": res["launches"],
            "on_demand": res.get("on_demand"), "apps": res.get("apps"),
            "l1_fill": res.get("l1_fill"), "host": host_info(),
            "per_rank": res["per_rank"], "value_per_gpu": res["value"] / world,
        }
        print(json.dumps(line))
    if world > 1:
        import torch.distributed as dist
        dist.destroy_process_group()
    return 0


def run_reference(args, world):
    """The oracle, as it stands, on the host cores (one bounded sample per step)."""
    cores = os.cpu_count() or 1
    import multiprocessing as mp
    ctx = mp.get_context("spawn")
    walkers, draws = 4096, 64  # ~0.3-0.6 s of oracle work per step (pool overhead < 1%)
    with ctx.Pool(cores) as pool:
        pool.map(_oracle_worker, [(0, 1, 1)] * cores)
        for _ in range(args.warmup):
            pool.map(_oracle_worker, [(c * walkers, walkers, draws) for c in range(cores)])
        t = time.perf_counter()
        for s in range(args.steps):
            pool.map(_oracle_worker, [((s * cores + c) * walkers, walkers, draws)
                                      for c in range(cores)])
        dt = time.perf_counter() - t
    labels = args.steps * cores * walkers * draws
    value = labels / dt / 1e9
    wl = "C5" if args.workload == "c5" else "C2"
    sample = (f"per step {cores * walkers * draws} labels of the {wl} workload (m=2^32, "
              f"l=l0=64): {cores} single-threaded oracle processes x {walkers} walkers x "
              f"{draws} draws")
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": dt * 1e3 / args.steps,
        "higher_is_better": True, "scaling": "strong" if args.workload == "c5" else "weak",
        "vs_baseline": None, "dtype": "u64",
        "data": "synthetic (SplitMix64 counter-hash seed bits, reading R9)",
        "config": {"workload": C5_WORKLOAD if args.workload == "c5" else WORKLOAD,
                   "number": "one 64-bit vertex label (the paper's unit)",
                   "parallelism": "host cores"},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line))
    return 0


if __name__ == "__main__":
    sys.exit(main())

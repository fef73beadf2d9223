"""B200-native expander-walk PRNG (Banerjee, Bahl & Kothapalli, IPDPS-W 2012).

Thin Python layer over the C ABI in include/prng.h (libggprng.so).  Every
step of the generator runs in the library's CUDA kernels; this module only
marshals arguments.  PyTorch supplies device memory and streams.

    from paper_conf_ipps_banerjeebk12_b200 import Generator
    g = Generator(walkers=1 << 20, seed=1)          # Alg.1 on the GPU
    out = torch.empty(1 << 30, dtype=torch.int32, device="cuda")
    g.fill(out)                                      # bulk Alg.2, 2^29 labels
"""
from __future__ import annotations

import ctypes
from contextlib import contextmanager

from . import _lib
from ._lib import (PRNG_BITS_CALLBACK, PRNG_BITS_GGCPU, PRNG_BITS_RANDR, PRNG_BITS_SPLITMIX,
                   PRNG_FMT_U32, PRNG_FMT_U64, PrngError, check)

__all__ = ["Generator", "PrngError", "PRNG_FMT_U32", "PRNG_FMT_U64", "PRNG_BITS_SPLITMIX",
           "PRNG_BITS_RANDR", "PRNG_BITS_CALLBACK", "PRNG_BITS_GGCPU", "params", "options"]


def params(m: int = 1 << 32, walk_len: int = 64, burnin_len: int = 64, degree: int = 7,
           variant: int = 0) -> _lib.prng_graph_params:
    p = _lib.prng_graph_params()
    check(_lib.prng_default_params(ctypes.byref(p)))
    p.m, p.walk_len, p.burnin_len, p.degree, p.variant = m, walk_len, burnin_len, degree, variant
    return p


def options(device: int = 0, walker_base: int = 0, epoch_draws: int = 16, host_threads: int = 0,
            bits_fn=None, bits_ctx=None, bit_source: int = 0) -> _lib.prng_options:
    o = _lib.prng_options()
    check(_lib.prng_default_options(ctypes.byref(o)))
    o.device, o.walker_base, o.epoch_draws, o.host_threads = device, walker_base, epoch_draws, host_threads
    o.bit_source = bit_source
    if bits_fn is not None:
        o.bit_source = PRNG_BITS_CALLBACK
        o.bits_fn = bits_fn
        o.bits_ctx = bits_ctx
    return o


def _stream_handle(stream) -> int:
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


def _fmt_of(t) -> int:
    import torch
    if t.dtype in (torch.int64, torch.uint64):
        return PRNG_FMT_U64
    if t.dtype in (torch.int32, torch.uint32):
        return PRNG_FMT_U32
    raise TypeError(f"output dtype must be a 32- or 64-bit integer, got {t.dtype}")


def _checked_count(t, n):
    """n (default: all) numbers fit the contiguous tensor t; the library
    writes n * itemsize bytes from t.data_ptr()."""
    if not t.is_contiguous():
        raise ValueError("output tensor must be contiguous")
    if n is None:
        return t.numel()
    if not 0 <= n <= t.numel():
        raise ValueError(f"n = {n} outside [0, {t.numel()}] for this output tensor")
    return n


class Generator:
    """One prng_t handle: W walkers of the 7-regular Gabber-Galil walk."""

    def __init__(self, walkers: int, seed: int, m: int = 1 << 32, walk_len: int = 64,
                 burnin_len: int = 64, device: int = 0, walker_base: int = 0,
                 epoch_draws: int = 16, host_threads: int = 0, bits_fn=None, variant: int = 0,
                 bit_source: int = 0):
        self._h = ctypes.c_void_p()
        self.walkers, self.seed, self.m, self.walk_len = walkers, seed, m, walk_len
        self._walker_base = walker_base
        self.device = device
        self._bits_fn = None
        if bits_fn is not None:
            # bits_fn(walker0, nwalkers, word0, nwords) -> numpy uint32 [nwords, nwalkers]
            import numpy as np

            def _cb(ctx, walker0, nwalkers, word0, nwords, out, pitch):
                a = np.asarray(bits_fn(walker0, nwalkers, word0, nwords), dtype=np.uint32)
                buf = np.ctypeslib.as_array(out, shape=((nwords - 1) * pitch + nwalkers,))
                for r in range(nwords):
                    buf[r * pitch:r * pitch + nwalkers] = a[r]
            self._bits_fn = _lib.PRNG_BITS_FN(_cb)
        p = params(m, walk_len, burnin_len, variant=variant)
        o = options(device, walker_base, epoch_draws, host_threads, self._bits_fn,
                    bit_source=bit_source)
        check(_lib.prng_create(ctypes.byref(self._h), ctypes.byref(p), walkers, seed,
                               ctypes.byref(o)), "prng_create")

    # -- bulk ---------------------------------------------------------------
    def fill(self, out, n: int | None = None, stream=None) -> None:
        """prng_fill: next n numbers into a CUDA tensor (int64 = labels, int32 = words)."""
        fmt = _fmt_of(out)
        if out.device.type != "cuda" or out.device.index != self.device:
            raise ValueError(f"fill: output must live on cuda:{self.device}, got {out.device}")
        n = _checked_count(out, n)
        check(_lib.prng_fill(self._h, out.data_ptr(), n, fmt, _stream_handle(stream)), "prng_fill")

    def fill_ptr(self, dev_ptr: int, n: int, fmt: int, stream: int) -> int:
        return _lib.prng_fill(self._h, dev_ptr, n, fmt, stream)

    def fill_host(self, out, n: int | None = None) -> None:
        """prng_fill_host: next n numbers into a host tensor / numpy array."""
        if hasattr(out, "data_ptr"):
            if out.device.type != "cpu":
                raise ValueError(f"fill_host: output must be host memory, got {out.device}")
            fmt, ptr = _fmt_of(out), out.data_ptr()
            n = _checked_count(out, n)
        else:
            if out.dtype.itemsize not in (4, 8) or out.dtype.kind not in "iu":
                raise TypeError(f"output dtype must be a 32- or 64-bit integer, got {out.dtype}")
            if not out.flags["C_CONTIGUOUS"]:
                raise ValueError("fill_host: output array must be C-contiguous")
            fmt = PRNG_FMT_U64 if out.dtype.itemsize == 8 else PRNG_FMT_U32
            ptr = out.ctypes.data
            n = out.size if n is None else n
            if not 0 <= n <= out.size:
                raise ValueError(f"fill_host: n = {n} outside [0, {out.size}]")
        check(_lib.prng_fill_host(self._h, ptr, n, fmt), "prng_fill_host")

    def prefetch(self, draws: int) -> None:
        check(_lib.prng_prefetch(self._h, draws), "prng_prefetch")

    def tell(self) -> int:
        v = ctypes.c_uint64()
        check(_lib.prng_tell(self._h, ctypes.byref(v)))
        return v.value

    def mark(self, stream=None) -> None:
        check(_lib.prng_mark(self._h, _stream_handle(stream)), "prng_mark")

    def rewind(self, stream=None) -> None:
        check(_lib.prng_rewind(self._h, _stream_handle(stream)), "prng_rewind")

    def save(self) -> bytes:
        n = ctypes.c_size_t()
        check(_lib.prng_state_size(self._h, ctypes.byref(n)))
        buf = ctypes.create_string_buffer(n.value)
        check(_lib.prng_save(self._h, buf, n.value), "prng_save")
        return buf.raw

    def load(self, blob: bytes) -> None:
        buf = ctypes.create_string_buffer(blob, len(blob))
        check(_lib.prng_load(self._h, buf, len(blob)), "prng_load")

    # -- on demand ----------------------------------------------------------
    def epoch_begin(self, active_walkers: int, draws: int, stream=None) -> None:
        check(_lib.prng_epoch_begin(self._h, active_walkers, draws, _stream_handle(stream)),
              "prng_epoch_begin")

    def epoch_begin_list(self, walkers, draws: int, stream=None) -> None:
        """prng_epoch_begin_list: window slot k holds walker walkers[k] (host uint32 array)."""
        import numpy as np
        ids = np.ascontiguousarray(walkers, dtype=np.uint32)
        check(_lib.prng_epoch_begin_list(self._h, ids.ctypes.data, ids.size, draws,
                                         _stream_handle(stream)), "prng_epoch_begin_list")

    def epoch_reserve(self, active_walkers: int, draws: int) -> None:
        """prng_epoch_reserve: pre-allocate both window slots up to this size."""
        check(_lib.prng_epoch_reserve(self._h, active_walkers, draws), "prng_epoch_reserve")

    def epoch_end(self, stream=None) -> None:
        check(_lib.prng_epoch_end(self._h, _stream_handle(stream)), "prng_epoch_end")

    @contextmanager
    def epoch(self, active_walkers: int, draws: int, stream=None):
        self.epoch_begin(active_walkers, draws, stream)
        try:
            yield self.view()
        finally:
            self.epoch_end(stream)

    def consume(self, threads: int, counts=None, uniform: int = 0, out=None, offsets=None,
                xor_out=None, stream=None) -> None:
        """gg_consume: synthetic on-demand demand (thread t calls prng_next on walker t)."""
        ptr = lambda t: None if t is None else t.data_ptr()
        check(_lib.gg_consume(self._h, threads, ptr(counts), uniform, ptr(out), ptr(offsets),
                              ptr(xor_out), _stream_handle(stream)), "gg_consume")

    def list_rank(self, succ, pred, head: int, removed_round=None, is_splitter=None, stream=None,
                  collective=None):
        """gg_list_rank: ranks (distance from head) of a linked list given as CUDA int32 arrays.

        collective: None (one GPU) or a dist.Collective (multi-GPU splitter exchange).
        Returns (rank tensor, info dict)."""
        import torch
        n = succ.numel()
        rank = torch.empty(n, dtype=torch.int32, device=succ.device)
        info = (ctypes.c_int64 * 8)()
        ptr = lambda t: None if t is None else t.data_ptr()
        coll = None if collective is None else ctypes.byref(collective.struct())
        check(_lib.gg_list_rank(self._h, n, succ.data_ptr(), pred.data_ptr(), head, rank.data_ptr(),
                                ptr(removed_round), ptr(is_splitter), info, coll,
                                _stream_handle(stream)),
              "gg_list_rank")
        keys = ("rounds", "reduced", "splitters", "draws", "phase1_us", "phase2_us", "phase3_us",
                "rounds2")
        return rank, {k: info[i] for i, k in enumerate(keys)}

    def mc_run(self, layers, photons_total: int, threads: int | None = None, n_top: float = 1.0,
               n_bottom: float = 1.0, threads_total: int | None = None, thread0: int | None = None,
               epoch_draws: int = 192, w_threshold: float = 1e-4, per_thread=None, stream=None):
        """gg_mc_run: Monte Carlo photon migration (Alg.4) driven by prng_next.

        layers: sequence of (n, mua, mus, g, d).  Returns a dict of fixed-point
        tallies (units 2^-32) and run statistics."""
        threads = self.walkers if threads is None else threads
        threads_total = threads if threads_total is None else threads_total
        thread0 = self._walker_base if thread0 is None else thread0
        arr = (_lib.gg_mc_layer * len(layers))(*[_lib.gg_mc_layer(*map(float, L)) for L in layers])
        cfg = _lib.gg_mc_config(arr, len(layers), n_top, n_bottom, photons_total, threads_total,
                                thread0, threads, epoch_draws, w_threshold)
        nt = 5 + len(layers)
        tal = (ctypes.c_int64 * nt)()
        stats = (ctypes.c_int64 * 7)()
        check(_lib.gg_mc_run(self._h, ctypes.byref(cfg), tal,
                             None if per_thread is None else per_thread.data_ptr(), stats,
                             _stream_handle(stream)), "gg_mc_run")
        names = ("launched", "specular", "R_d", "T_t", "terminated")
        out = {k: tal[i] for i, k in enumerate(names)}
        out["absorbed"] = [tal[i] for i in range(5, nt)]
        out["tallies"] = [tal[i] for i in range(nt)]
        for i, k in enumerate(("photons", "draws", "epochs", "interactions", "kernel_us", "total_us",
                               "walker_epochs_fed")):
            out[k] = stats[i]
        return out

    def view(self) -> _lib.prng_view:
        v = _lib.prng_view()
        check(_lib.prng_device_view(self._h, ctypes.byref(v), ctypes.sizeof(v)), "prng_device_view")
        return v

    def check(self) -> int:
        return _lib.prng_check(self._h)

    def stats(self) -> dict:
        s = _lib.prng_stats()
        check(_lib.prng_get_stats(self._h, ctypes.byref(s)))
        return {k: getattr(s, k) for k, _ in s._fields_}

    @property
    def handle(self) -> int:
        return self._h.value

    def close(self) -> None:
        if self._h:
            _lib.prng_destroy(self._h)
            self._h = ctypes.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

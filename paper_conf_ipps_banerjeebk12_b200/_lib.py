"""ctypes binding to libggprng.so (argument marshalling only).

Function names match include/prng.h.  There is no fallback: if the native
library is missing or fails to load, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libggprng.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        f"{LIB_PATH} is missing: build it with `python paper_conf_ipps_banerjeebk12_b200/build.py` "
        "(or __graft_entry__.build()); there is no CPU fallback")

_L = ctypes.CDLL(LIB_PATH)

c_int = ctypes.c_int
u32 = ctypes.c_uint32
u64 = ctypes.c_uint64
vp = ctypes.c_void_p
sz = ctypes.c_size_t

PRNG_OK = 0
PRNG_E_INVALID = -1
PRNG_E_UNSUPPORTED = -2
PRNG_E_NOMEM = -3
PRNG_E_CUDA = -4
PRNG_E_OVERRUN = -5
PRNG_E_STATE = -6
PRNG_FMT_U64 = 0
PRNG_FMT_U32 = 1
PRNG_BITS_SPLITMIX = 0
PRNG_BITS_RANDR = 1
PRNG_BITS_CALLBACK = 2
PRNG_BITS_GGCPU = 3

PRNG_BITS_FN = ctypes.CFUNCTYPE(None, vp, u64, u64, u64, u32, ctypes.POINTER(ctypes.c_uint32), u64)


class prng_graph_params(ctypes.Structure):
    _fields_ = [("m", u64), ("degree", u32), ("walk_len", u32), ("burnin_len", u32),
                ("variant", u32)]


class prng_options(ctypes.Structure):
    _fields_ = [("device", c_int), ("walker_base", u64), ("epoch_draws", u32),
                ("host_threads", u32), ("bit_source", u32), ("bits_fn", PRNG_BITS_FN),
                ("bits_ctx", vp)]


class prng_stats(ctypes.Structure):
    _fields_ = [("labels_generated", u64), ("bits_bytes_fed", u64), ("h2d_bytes", u64),
                ("d2h_bytes", u64), ("kernel_launches", u64), ("feed_seconds", ctypes.c_double),
                ("feed_pace_mbs", u32), ("_reserved", u32)]


class gg_mc_layer(ctypes.Structure):
    _fields_ = [("n", ctypes.c_double), ("mua", ctypes.c_double), ("mus", ctypes.c_double),
                ("g", ctypes.c_double), ("d", ctypes.c_double)]


class gg_mc_config(ctypes.Structure):
    _fields_ = [("layers", ctypes.POINTER(gg_mc_layer)), ("nlayers", c_int),
                ("n_top", ctypes.c_double), ("n_bottom", ctypes.c_double),
                ("photons_total", u64), ("threads_total", u64), ("thread0", u64),
                ("threads", u64), ("epoch_draws", u32), ("w_threshold", ctypes.c_double)]


GG_ALLGATHER_FN = ctypes.CFUNCTYPE(c_int, vp, vp, vp, sz)
GG_ALLREDUCE_I32_FN = ctypes.CFUNCTYPE(c_int, vp, vp, sz)


class gg_collective(ctypes.Structure):
    _fields_ = [("rank", c_int), ("world", c_int), ("allgather", GG_ALLGATHER_FN),
                ("allreduce_i32", GG_ALLREDUCE_I32_FN), ("ctx", vp)]


class prng_view(ctypes.Structure):
    """Mirror of struct prng_view (include/prng_device.cuh)."""
    _fields_ = [("bits", vp), ("wmap", vp), ("x", vp), ("y", vp), ("j", vp), ("flags", vp), ("pitch", u64),
                ("m", u64), ("J0", u32), ("D", u32), ("Wv", u32), ("R", u32), ("l", u32),
                ("log2m", u32), ("pow2", u32), ("variant", u32), ("l0", u32),
                ("_pad", u32), ("tab", vp)]


_SIGS = {
    "prng_version": (c_int, []),
    "prng_strerror": (ctypes.c_char_p, [c_int]),
    "prng_default_params": (c_int, [ctypes.POINTER(prng_graph_params)]),
    "prng_default_options": (c_int, [ctypes.POINTER(prng_options)]),
    "prng_create": (c_int, [ctypes.POINTER(vp), ctypes.POINTER(prng_graph_params), u64, u64,
                            ctypes.POINTER(prng_options)]),
    "prng_fill": (c_int, [vp, vp, u64, c_int, vp]),
    "prng_fill_host": (c_int, [vp, vp, u64, c_int]),
    "prng_prefetch": (c_int, [vp, u64]),
    "prng_tell": (c_int, [vp, ctypes.POINTER(u64)]),
    "prng_mark": (c_int, [vp, vp]),
    "prng_rewind": (c_int, [vp, vp]),
    "prng_state_size": (c_int, [vp, ctypes.POINTER(sz)]),
    "prng_save": (c_int, [vp, vp, sz]),
    "prng_load": (c_int, [vp, vp, sz]),
    "prng_epoch_begin": (c_int, [vp, u64, u32, vp]),
    "prng_epoch_begin_list": (c_int, [vp, vp, u64, u32, vp]),
    "prng_epoch_end": (c_int, [vp, vp]),
    "prng_epoch_reserve": (c_int, [vp, ctypes.c_uint64, ctypes.c_uint32]),
    "prng_device_view": (c_int, [vp, vp, sz]),
    "prng_check": (c_int, [vp]),
    "prng_get_stats": (c_int, [vp, ctypes.POINTER(prng_stats)]),
    "prng_destroy": (c_int, [vp]),
    # include/gg_apps.h
    "gg_consume": (c_int, [vp, u64, vp, u32, vp, vp, vp, vp]),
    "gg_list_rank": (c_int, [vp, ctypes.c_int64, vp, vp, ctypes.c_int64, vp, vp, vp, vp,
                             ctypes.POINTER(gg_collective), vp]),
    "gg_mc_run": (c_int, [vp, ctypes.POINTER(gg_mc_config), vp, vp, vp, vp]),
}

for _name, (_res, _args) in _SIGS.items():
    _fn = getattr(_L, _name)
    _fn.restype = _res
    _fn.argtypes = _args
    globals()[_name] = _fn

EXPORTED = tuple(_SIGS)


class PrngError(RuntimeError):
    def __init__(self, status: int, where: str = ""):
        self.status = status
        msg = prng_strerror(status).decode()
        super().__init__(f"{where}: {msg} ({status})" if where else f"{msg} ({status})")


def check(status: int, where: str = "") -> int:
    if status != PRNG_OK:
        raise PrngError(status, where)
    return status


def lib():
    return _L

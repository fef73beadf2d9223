"""CPU oracle for the expander-walk PRNG (Banerjee, Bahl & Kothapalli, IPDPS-W 2012).

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and the
``cpu_baseline`` / ``--impl reference`` legs of ``bench.py`` may import this
package.  The product package ``paper_conf_ipps_banerjeebk12_b200`` never
imports it and shares no code with it.

The arithmetic lives in plain single-threaded C (``gg_oracle.c``,
``lr_oracle.c``, ``mc_oracle.c``); this module only compiles and loads it and
marshals numpy arrays.  Every C function cites the PAPER.md passage it follows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SOURCES = ["gg_oracle.c", "lr_oracle.c", "mc_oracle.c"]
_LIB_PATH = os.path.join(_HERE, "libggoracle.so")
_lock = threading.Lock()
_lib = None

u64 = ctypes.c_uint64
u32 = ctypes.c_uint32
i32 = ctypes.c_int32
i64 = ctypes.c_int64
f64 = ctypes.c_double
P = ctypes.c_void_p


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (plain -O2, no fast-math, no FP contraction)."""
    srcs = [os.path.join(_HERE, s) for s in _SOURCES if os.path.exists(os.path.join(_HERE, s))]
    newest = max(os.path.getmtime(s) for s in srcs)
    if not force and os.path.exists(_LIB_PATH) and os.path.getmtime(_LIB_PATH) >= newest:
        return _LIB_PATH
    tmp = _LIB_PATH + f".tmp{os.getpid()}"
    cmd = ["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-ffp-contract=off",
           "-fno-fast-math", "-Wall", "-o", tmp] + srcs + ["-lm"]
    subprocess.check_call(cmd)
    os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB_PATH)
            sig = {
                "or_mix64": (u64, [u64]),
                "or_stream_word64": (u64, [u64, u64, u64]),
                "or_stream_word32": (u32, [u64, u64, u64]),
                "or_words_per_walk": (u32, [u32]),
                "or_bits3": (ctypes.c_int, [P, u32]),
                "or_walk": (None, [u64, P, P, P, u32]),
                "or_label": (u64, [u64, u64, u64]),
                "or_draw_word_index": (u64, [u32, u32, u64, u32]),
                "or_walker_init": (ctypes.c_int, [u64, u32, u64, u64, P, P]),
                "or_walker_draw": (u64, [u64, u32, u32, u64, u64, u64, P, P]),
                "or_bulk": (ctypes.c_int, [u64, u32, u32, u64, u64, u64, u64, P]),
                "or_walker_draws": (ctypes.c_int, [u64, u32, u32, u64, u64, u64, u64, P]),
                "or_sigma_array": (None, [u64, ctypes.c_int, P, P, P, P, u64]),
                "or_stream_block": (None, [u64, u64, u64, u64, u32, P]),
                "or_sigma_inv": (None, [u64, ctypes.c_int, u64, u64, P, P]),
                "or_rand_r": (ctypes.c_int32, [P]),
                "or_stream_word32_randr": (u32, [u64, u64, u64]),
                "or_stream_word32_ggcpu": (u32, [u64, u64, u64]),
                "or_set_bit_source": (None, [ctypes.c_int]),
                "or_walk_bipartite": (None, [u64, P, P, P, u32, u64]),
                "or_walker_init_v": (ctypes.c_int, [u64, u32, u32, u64, u64, P, P]),
                "or_walker_draw_v": (u64, [u64, u32, u32, u32, u64, u64, u64, P, P]),
                "or_bulk_v": (ctypes.c_int, [u64, u32, u32, u32, u64, u64, u64, u64, P]),
            }
            for name, (res, args) in sig.items():
                fn = getattr(L, name)
                fn.restype = res
                fn.argtypes = args
            _bind_optional(L)
            _lib = L
    return _lib


def _bind_optional(L):
    """Signatures of the application oracles (list ranking, Monte Carlo)."""
    opt = {
        "or_lr_rank_seq": (ctypes.c_int, [i64, P, i64, P]),
        "or_lr_run": (ctypes.c_int, [u64, u32, u32, u64, i64, P, P, i64, i64, P, P, P, P]),
        "or_mc_run": (ctypes.c_int, [P, ctypes.c_int, f64, f64, u64, u32, u32, u64, u64, u64, u64,
                                     u64, u32, f64, P, P, P]),
        "or_mc_xi": (f64, [u64]),
        "or_mc_hg": (f64, [f64, f64]),
        "or_mc_fresnel": (f64, [f64, f64, f64, P]),
        "or_mc_q": (u64, [f64]),
        "or_mc_refract": (None, [f64, f64, f64, P, P, P]),
        "or_mc_spin": (None, [f64, f64, f64, P, P, P]),
    }
    for name, (res, args) in opt.items():
        fn = getattr(L, name, None)
        if fn is not None:
            fn.restype = res
            fn.argtypes = args


def _ptr(a: np.ndarray):
    return ctypes.c_void_p(a.ctypes.data)


# ----------------------------------------------------------------------------
# Thin numpy wrappers (argument marshalling only).
# ----------------------------------------------------------------------------

def mix64(z: int) -> int:
    return int(lib().or_mix64(z))


def stream_word32(seed: int, t: int, k: int) -> int:
    return int(lib().or_stream_word32(seed, t, k))


def stream_word64(seed: int, t: int, c: int) -> int:
    return int(lib().or_stream_word64(seed, t, c))


def words_per_walk(nsteps: int) -> int:
    return int(lib().or_words_per_walk(nsteps))


def sigma(m: int, k: int, x, y):
    """sigma_k applied elementwise to arrays x, y (uint64)."""
    x = np.ascontiguousarray(x, dtype=np.uint64)
    y = np.ascontiguousarray(y, dtype=np.uint64)
    nx = np.empty_like(x)
    ny = np.empty_like(y)
    lib().or_sigma_array(m, k, _ptr(x), _ptr(y), _ptr(nx), _ptr(ny), x.size)
    return nx, ny


def bits3(rec, i: int) -> int:
    rec = np.ascontiguousarray(rec, dtype=np.uint32)
    return int(lib().or_bits3(_ptr(rec), i))


def walk(m: int, x: int, y: int, rec, nsteps: int):
    """One walk of nsteps with an explicit bit record (user-supplied bits)."""
    rec = np.ascontiguousarray(rec, dtype=np.uint32)
    xs = np.array([x], dtype=np.uint64)
    ys = np.array([y], dtype=np.uint64)
    lib().or_walk(m, _ptr(xs), _ptr(ys), _ptr(rec), nsteps)
    return int(xs[0]), int(ys[0])


def label(m: int, x: int, y: int) -> int:
    return int(lib().or_label(m, x, y))


def walker_init(m: int, l0: int, seed: int, t: int):
    xs = np.zeros(1, dtype=np.uint64)
    ys = np.zeros(1, dtype=np.uint64)
    rc = lib().or_walker_init(m, l0, seed, t, _ptr(xs), _ptr(ys))
    if rc != 0:
        raise ValueError("or_walker_init failed")
    return int(xs[0]), int(ys[0])


def walker_draws(m: int, l: int, l0: int, seed: int, t: int, j0: int, nd: int) -> np.ndarray:
    out = np.empty(nd, dtype=np.uint64)
    rc = lib().or_walker_draws(m, l, l0, seed, t, j0, nd, _ptr(out))
    if rc != 0:
        raise ValueError("or_walker_draws failed")
    return out


def bulk(m: int, l: int, l0: int, seed: int, W: int, g0: int, n: int) -> np.ndarray:
    out = np.empty(n, dtype=np.uint64)
    rc = lib().or_bulk(m, l, l0, seed, W, g0, n, _ptr(out))
    if rc != 0:
        raise ValueError("or_bulk failed")
    return out


class bit_source:
    """Context manager selecting the oracle's seed-bit stream (0 = SplitMix64, 1 = rand_r)."""

    def __init__(self, src: int):
        self.src = src

    def __enter__(self):
        lib().or_set_bit_source(self.src)

    def __exit__(self, *exc):
        lib().or_set_bit_source(0)


def sigma_inv(m: int, k: int, x: int, y: int):
    nx = np.zeros(1, np.uint64)
    ny = np.zeros(1, np.uint64)
    lib().or_sigma_inv(m, k, x, y, _ptr(nx), _ptr(ny))
    return int(nx[0]), int(ny[0])


def bulk_v(m: int, l: int, l0: int, variant: int, seed: int, W: int, g0: int, n: int) -> np.ndarray:
    out = np.empty(n, dtype=np.uint64)
    rc = lib().or_bulk_v(m, l, l0, variant, seed, W, g0, n, _ptr(out))
    if rc != 0:
        raise ValueError("or_bulk_v failed")
    return out


def stream_block(seed: int, t0: int, count: int, k0: int, nwords: int) -> np.ndarray:
    out = np.empty((nwords, count), dtype=np.uint32)
    lib().or_stream_block(seed, t0, count, k0, nwords, _ptr(out))
    return out


def lr_rank_seq(succ, head: int) -> np.ndarray:
    """Ranks by walking the list from the head (the definition, R17)."""
    succ = np.ascontiguousarray(succ, dtype=np.int32)
    rank = np.full(succ.size, -1, dtype=np.int32)
    reached = lib().or_lr_rank_seq(succ.size, _ptr(succ), head, _ptr(rank))
    if reached != succ.size:
        raise ValueError("not a single list")
    return rank


def lr_run(succ, pred, head: int, seed: int, m: int = 1 << 32, l: int = 64, l0: int = 64,
           max_rounds: int = 1000):
    """Sequential replica of Alg.3 + Helman-JaJa + re-insertion (lr_oracle.c)."""
    succ = np.ascontiguousarray(succ, dtype=np.int32)
    pred = np.ascontiguousarray(pred, dtype=np.int32)
    n = succ.size
    rank = np.full(n, -1, dtype=np.int32)
    removed = np.empty(n, dtype=np.int32)
    spl = np.empty(n, dtype=np.int32)
    info = np.zeros(4, dtype=np.int64)
    rc = lib().or_lr_run(m, l, l0, seed, n, _ptr(succ), _ptr(pred), head, max_rounds,
                         _ptr(rank), _ptr(removed), _ptr(spl), _ptr(info))
    if rc != 0:
        raise MemoryError("or_lr_run")
    return {"rank": rank, "removed_round": removed, "is_splitter": spl.astype(bool),
            "rounds": int(info[0]), "reduced": int(info[1]), "splitters": int(info[2]),
            "draws": int(info[3])}


# ---------------------------------------------------------------- Monte Carlo
MC_TALLY_NAMES = ("launched", "specular", "R_d", "T_t", "terminated")

# R19: MCML's sample slab (n, mua [1/cm], mus [1/cm], g, d [cm]); ambient n = 1.
MC_LAYERS_R19 = ((1.37, 1.0, 100.0, 0.9, 0.1), (1.37, 1.0, 10.0, 0.0, 0.1), (1.37, 2.0, 10.0, 0.7, 0.2))


def mc_run(layers=MC_LAYERS_R19, n_top=1.0, n_bottom=1.0, seed=0x5EED0004, walker0=0,
           nthreads=64, photons_total=256, threads_total=None, D=192, w_th=1e-4,
           m=1 << 32, l=64, l0=64, per_thread=False):
    """Sequential replica of the GPU photon-migration run (mc_oracle.c)."""
    layers = np.ascontiguousarray(np.array(layers, dtype=np.float64).reshape(-1, 5))
    nl = layers.shape[0]
    threads_total = nthreads if threads_total is None else threads_total
    tal = np.zeros(5 + nl, dtype=np.int64)
    pt = np.zeros((nthreads, 5 + nl), dtype=np.int64) if per_thread else None
    stats = np.zeros(4, dtype=np.int64)
    rc = lib().or_mc_run(_ptr(layers), nl, n_top, n_bottom, m, l, l0, seed, walker0, nthreads,
                         photons_total, threads_total, D, w_th, _ptr(tal),
                         None if pt is None else _ptr(pt), _ptr(stats))
    if rc != 0:
        raise ValueError("or_mc_run")
    out = {k: int(tal[i]) for i, k in enumerate(MC_TALLY_NAMES)}
    out["absorbed"] = [int(v) for v in tal[5:]]
    out["tallies"] = tal
    out["photons"], out["draws"], out["epochs"], out["interactions"] = (int(v) for v in stats)
    if per_thread:
        out["per_thread"] = pt
    return out


def mc_hg(g: float, xi: float) -> float:
    return float(lib().or_mc_hg(g, xi))


def mc_fresnel(n1: float, n2: float, ca1: float):
    ca2 = np.zeros(1)
    r = lib().or_mc_fresnel(n1, n2, ca1, _ptr(ca2))
    return float(r), float(ca2[0])


def mc_refract(n1: float, n2: float, ca2: float, u):
    """Transmitted direction (or_mc_refract) of direction u = (ux, uy, uz)."""
    v = [np.array([float(c)]) for c in u]
    lib().or_mc_refract(n1, n2, ca2, _ptr(v[0]), _ptr(v[1]), _ptr(v[2]))
    return tuple(float(c[0]) for c in v)


def mc_spin(g: float, xi_theta: float, xi_psi: float, u):
    """Direction after one scattering event (or_mc_spin) of direction u."""
    v = [np.array([float(c)]) for c in u]
    lib().or_mc_spin(g, xi_theta, xi_psi, _ptr(v[0]), _ptr(v[1]), _ptr(v[2]))
    return tuple(float(c[0]) for c in v)

"""GPU Monte Carlo photon migration (gg_mc_run) vs the CPU oracle.

Config C4 (BASELINE.json configs[3]): the paper's Monte Carlo simulation with
~2^32 draws on demand (2^20 threads x 20 photons, ~200 draws per photon),
partial sums combined by integer allreduce.  North-star tolerance: agree
within 1e-9 relative; with fixed-point tallies the expected result is exact
equality (a libm ulp difference at a decision threshold is the only way to
differ, probability ~1e-5 per run).
"""
import numpy as np
import pytest

import oracle as O

pytestmark = pytest.mark.gpu

R19 = O.MC_LAYERS_R19


def gpu_mc(threads, P, layers=R19, seed=0x5EED0004, walker_base=0, threads_total=None,
           D=192, n_top=1.0, n_bottom=1.0, per_thread=False):
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    g = Generator(walkers=threads, seed=seed, walker_base=walker_base)
    pt = None
    if per_thread:
        pt = torch.zeros(threads * (5 + len(layers)), dtype=torch.int64, device="cuda")
    r = g.mc_run(layers, P, threads=threads, threads_total=threads_total, epoch_draws=D,
                 n_top=n_top, n_bottom=n_bottom, per_thread=pt)
    if per_thread:
        r["per_thread"] = pt.view(threads, -1).cpu().numpy()
    g.close()
    return r


def assert_tallies_match(got, want):
    got = np.array(got, dtype=np.int64)
    want = np.array(want, dtype=np.int64)
    if not np.array_equal(got, want):
        rel = np.abs(got - want) / np.maximum(np.abs(want), 1)
        assert rel.max() <= 1e-9, (got, want)


def test_small_r19_exact_parity():
    T, P = 4096, 16384
    g = gpu_mc(T, P, per_thread=True)
    o = O.mc_run(nthreads=T, photons_total=P, D=192, seed=0x5EED0004, per_thread=True)
    assert_tallies_match(g["tallies"], o["tallies"])
    assert g["photons"] == P and g["epochs"] >= o["epochs"]
    assert g["interactions"] == o["interactions"]
    assert np.array_equal(g["per_thread"], o["per_thread"])
    t = g["tallies"]
    assert t[0] == sum(t[1:])  # exact conservation


@pytest.mark.parametrize("layers,n_top,n_bottom", [
    ([(1.5, 0.5, 20.0, 0.8, 0.05)], 1.0, 1.0),                       # mismatched: Fresnel, TIR
    ([(1.0, 2.0, 0.0, 0.0, 0.5)], 1.0, 1.0),                         # pure absorber
    ([(1.4, 1.0, 50.0, -0.3, 0.02), (1.33, 0.2, 5.0, 0.95, 0.3)], 1.0, 1.5),
])
def test_other_slabs_exact_parity(layers, n_top, n_bottom):
    T, P = 2048, 6000
    g = gpu_mc(T, P, layers=layers, n_top=n_top, n_bottom=n_bottom, D=48)
    o = O.mc_run(layers=layers, n_top=n_top, n_bottom=n_bottom, nthreads=T, photons_total=P,
                 D=48, seed=0x5EED0004)
    assert_tallies_match(g["tallies"], o["tallies"])


def test_shards_sum_to_single_run():
    # multi-GPU shape on one GPU: two walker shards with disjoint global ids
    T, P = 4096, 9000
    whole = gpu_mc(T, P)
    a = gpu_mc(T // 2, P, walker_base=0, threads_total=T)
    b = gpu_mc(T // 2, P, walker_base=T // 2, threads_total=T)
    assert np.array_equal(np.array(a["tallies"]) + np.array(b["tallies"]), np.array(whole["tallies"]))


def test_c4_full_size_conservation_and_sampled_parity():
    T = 1 << 20
    P = 20 * T
    g = gpu_mc(T, P, per_thread=True)
    t = g["tallies"]
    assert t[0] == sum(t[1:])
    assert g["photons"] == P
    assert g["draws"] > 2 ** 31.5   # ~2^32 draws on demand
    W = t[0]
    assert 0.20 < t[2] / W < 0.28 and 0.07 < t[3] / W < 0.13   # R_d, T_t of the R19 slab
    pt = g["per_thread"]
    assert np.array_equal(pt.sum(axis=0), np.array(t))
    for tg in list(range(0, T, T // 48)) + [T - 1]:
        o = O.mc_run(nthreads=1, walker0=tg, threads_total=T, photons_total=P, D=192,
                     seed=0x5EED0004)
        assert np.array_equal(pt[tg], o["tallies"]), tg


@pytest.mark.parametrize("T,P,D", [(1, 1, 3), (1, 5, 6), (100, 7, 3), (33, 1000, 9), (4096, 4095, 192)])
def test_degenerate_sizes_exact_parity(T, P, D):
    """Fewer photons than threads (idle threads), one thread, tiny epochs
    (one iteration per epoch), photon counts not divisible by threads."""
    g = gpu_mc(T, P, D=D, per_thread=True)
    o = O.mc_run(nthreads=T, photons_total=P, D=D, seed=0x5EED0004, per_thread=True)
    assert_tallies_match(g["tallies"], o["tallies"])
    assert g["photons"] == P
    assert np.array_equal(g["per_thread"], o["per_thread"])

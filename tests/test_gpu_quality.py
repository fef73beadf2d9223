"""Statistical quality of full-size GPU output (SURVEY §8(f) f4, P7-P9 at scale).

The paper's batteries (DIEHARD, TestU01; §IV-B Tables II-III) are not
available offline; these are the oracle's chi-square / serial / gap tests
run on 2^26 numbers of the C2 generator (m = 2^32) computed on the GPU,
with a negative control: with l = 16 steps per number the serial test on
(x mod 2, y mod 2) of consecutive draws must fail (the parity chain mixes at
rate 3/4 per step, P4: divergence ~2 (3/4)^32 ~ 2e-4 per pair).
"""
import numpy as np
import pytest
from scipy import stats

pytestmark = pytest.mark.gpu
ALPHA = 1e-3


def gen(l, n_draws=64, W=1 << 20, seed=0x5EED0002):
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    g = Generator(walkers=W, seed=seed, walk_len=l)
    o = torch.empty(W * n_draws, dtype=torch.int64, device="cuda")
    g.fill(o)
    torch.cuda.synchronize()
    return o.view(n_draws, W)


def chi2_p(counts, expected):
    counts = counts.double().cpu().numpy()
    chi = ((counts - expected) ** 2 / expected).sum()
    return stats.chi2.sf(chi, counts.size - 1)


def test_bytes_bits_serial_gap_l64():
    import torch
    z = gen(64)
    flat = z.reshape(-1)
    N = flat.numel()
    # each byte of the label uniform over 256 values
    for b in range(8):
        v = (flat >> (8 * b)) & 0xFF
        assert chi2_p(torch.bincount(v, minlength=256), N / 256) > ALPHA, b
    # each of the 64 bits fair within 5 sigma
    for bit in range(64):
        ones = ((flat >> bit) & 1).sum().item()
        assert abs(ones - N / 2) < 5 * 0.5 * N ** 0.5, bit
    # serial: consecutive draws of the same walker, parity and top-bit projections
    a, c = z[:-1].reshape(-1), z[1:].reshape(-1)
    par = lambda v: (v & 1) | (((v >> 32) & 1) << 1)
    cell = par(a) * 4 + par(c)
    assert chi2_p(torch.bincount(cell, minlength=16), cell.numel() / 16) > ALPHA
    top = lambda v: (((v >> 30) & 3) | (((v >> 62) & 3) << 2))
    cell = top(a) * 16 + top(c)
    assert chi2_p(torch.bincount(cell, minlength=256), cell.numel() / 256) > ALPHA
    # gap test on the top bit along each walker's sequence (first 4096 walkers)
    bits = ((z[:, :4096] >> 63) & 1).T.reshape(-1).cpu().numpy()
    idx = np.flatnonzero(bits)
    gaps = np.minimum(np.diff(idx) - 1, 10)
    counts = np.bincount(gaps, minlength=11).astype(float)
    p = np.array([0.5 ** (g + 1) for g in range(10)] + [0.5 ** 10])
    chi = ((counts - p * gaps.size) ** 2 / (p * gaps.size)).sum()
    assert stats.chi2.sf(chi, 10) > ALPHA


def test_negative_control_l16_serial_parity_fails():
    import torch
    z = gen(16, n_draws=16)
    a, c = z[:-1].reshape(-1), z[1:].reshape(-1)
    par = lambda v: (v & 1) | (((v >> 32) & 1) << 1)
    cell = par(a) * 4 + par(c)
    assert chi2_p(torch.bincount(cell, minlength=16), cell.numel() / 16) < 1e-10


def test_battery_on_gpu_output():
    """SmallCrush-style battery (tests/battery.py) on 2^23 labels of the C2
    generator computed on the GPU, bulk order and walker-major order."""
    import battery as B
    z = gen(64, n_draws=64, W=1 << 17).cpu().numpy()  # [draw, walker] int64
    for name, arr in (("bulk", z), ("walker-major", z.T.copy())):
        res = B.run(np.ascontiguousarray(arr).reshape(-1).view(np.uint32))
        bad = {k: v for k, v in res.items() if v < 1e-4}
        assert not bad, (name, bad)


def test_battery_negative_control_l1_on_gpu():
    import battery as B
    z = gen(1, n_draws=1024, W=1 << 12).cpu().numpy()
    res = B.run(np.ascontiguousarray(z.T).reshape(-1).view(np.uint32))
    assert sum(v < 1e-10 for v in res.values()) >= 3, res


def test_nist_sp800_22_on_gpu_output():
    """NIST SP 800-22 subset (tests/nist.py) on 16 sequences of 10^6 bits of
    C2 output computed on the GPU, bulk and walker-major order.  NIST's
    acceptance rule: the proportion of sequences passing at alpha = 0.01 must
    exceed 0.99 - 3 sqrt(0.99 * 0.01 / k); for k = 16 at most one failure is
    expected, allow three (P(>= 4 of 16) ~ 2e-6 per test)."""
    import nist as N
    z = gen(64, n_draws=16, W=1 << 16).cpu().numpy()  # 2^20 labels = 2^26 bits
    for name, arr in (("bulk", z), ("walker-major", z.T.copy())):
        bits = N.bits_of_words(np.ascontiguousarray(arr).reshape(-1).view(np.uint32))
        fails = {}
        for s in range(16):
            for k, v in N.run(bits[s * 1_000_000:(s + 1) * 1_000_000]).items():
                fails[k] = fails.get(k, 0) + (v < 0.01)
        assert max(fails.values()) <= 3, (name, fails)


def test_crush_style_on_gpu_output():
    """Crush-style tests (tests/battery_crush.py) on 2^23 labels of the C2
    generator computed on the GPU, bulk and walker-major order."""
    import battery_crush as C
    z = gen(64, n_draws=64, W=1 << 17).cpu().numpy()
    for name, arr in (("bulk", z), ("walker-major", z.T.copy())):
        res = C.run(np.ascontiguousarray(arr).reshape(-1).view(np.uint32))
        bad = {k: v for k, v in res.items() if v < 1e-4}
        assert not bad, (name, bad)


def test_c1_chi_square_on_gpu_output():
    """BASELINE C1 ("tiny expander (m=2^8), 1024 walkers, 2^20 numbers - GPU vs
    CPU oracle bit-exact, chi-square check"): the 2^20 labels computed on the
    GPU are equidistributed over the m^2 = 65536 vertices (chi-square, 65535
    dof), and so are the pairs (x mod 16, y mod 16) of consecutive draws of a
    walker (serial test, 65535 dof over 16^4 cells)."""
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, n = 1024, 1 << 20
    g = Generator(walkers=W, seed=0x5EED0001, m=256)
    o = torch.empty(n, dtype=torch.int64, device="cuda")
    g.fill(o)
    lab = o.cpu()
    p1 = chi2_p(torch.bincount(lab, minlength=65536), n / 65536)
    z = lab.view(n // W, W)
    x, y = z % 256, z // 256
    cell = ((x[:-1] % 16) * 16 + y[:-1] % 16) * 256 + (x[1:] % 16) * 16 + y[1:] % 16
    p2 = chi2_p(torch.bincount(cell.reshape(-1), minlength=65536), cell.numel() / 65536)
    assert p1 > ALPHA and p2 > ALPHA, (p1, p2)
    g.close()


def test_crush_scale_battery_small():
    """The 15 streaming statistics of tests/battery_gpu.py (the ones
    tools/battery_big.py runs at 2^33 words, profiles/r02_battery.json) at
    2^26 words: l = 64 passes all 15 in bulk and walker-major order, the
    l = 1 walk fails several (§IV-B Table III)."""
    import os
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    sys.path.insert(0, os.path.join(root, "tools"))
    import battery_big as BB
    import battery_gpu as G

    def tests():
        return G.crush_scale_tests(rank300_matrices=1 << 11, samples_n=1 << 22)
    for r in (BB.run_stream(BB.gen_chunks(1 << 25, 1 << 20), tests()),
              BB.run_stream(BB.gen_chunks(1 << 25, 4096, walker_major=True), tests())):
        assert r["failed"] == [], r
        assert r["passed"] == "15/15"
    bad = BB.run_stream(BB.gen_chunks(1 << 24, 1 << 20, walk_len=1), tests())
    assert len(bad["failed"]) >= 3, bad

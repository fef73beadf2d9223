"""Stream semantics of the C ABI (include/prng.h "stream" arguments).

prng_fill / prng_epoch_* / gg_consume enqueue their device work on the
caller's stream and return: work the caller enqueued earlier on that stream
runs before, work enqueued later runs after, and handles used on different
streams do not interfere.  Checked against the oracle with no device-wide
synchronisation between the enqueued steps.
"""
import numpy as np
import pytest

import oracle as O

pytestmark = pytest.mark.gpu
M32 = 1 << 32


def test_fill_is_ordered_on_the_callers_stream():
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, D, seed = 3000, 40, 31
    g = Generator(walkers=W, seed=seed)
    g.prefetch(D)  # K-mode: the fill is kernels only, fully asynchronous
    s = torch.cuda.Stream()
    out = torch.empty(W * D, dtype=torch.int64, device="cuda")
    with torch.cuda.stream(s):
        big = torch.empty(1 << 28, dtype=torch.float32, device="cuda")
        for _ in range(4):  # keep the stream busy before the fill
            big.mul_(1.0001)
        out.fill_(-1)
        g.fill(out, stream=s)
        snap = out.clone()  # enqueued after the fill on the same stream
    s.synchronize()
    want = O.bulk(M32, 64, 64, seed, W, 0, W * D)
    assert np.array_equal(snap.cpu().numpy().view(np.uint64), want)
    g.close()


def test_two_handles_on_two_streams():
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, D = 2048, 24
    ga, gb = Generator(walkers=W, seed=1), Generator(walkers=W, seed=2, m=256)
    sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
    oa = torch.empty(W * D, dtype=torch.int64, device="cuda")
    ob = torch.empty(W * D, dtype=torch.int64, device="cuda")
    half = W * D // 2 + 5
    with torch.cuda.stream(sa):
        ga.fill(oa[:half], stream=sa)
    with torch.cuda.stream(sb):
        gb.fill(ob[:half], stream=sb)
    with torch.cuda.stream(sa):
        ga.fill(oa[half:], stream=sa)
    with torch.cuda.stream(sb):
        gb.fill(ob[half:], stream=sb)
    sa.synchronize()
    sb.synchronize()
    assert np.array_equal(oa.cpu().numpy().view(np.uint64), O.bulk(M32, 64, 64, 1, W, 0, W * D))
    assert np.array_equal(ob.cpu().numpy().view(np.uint64), O.bulk(256, 64, 64, 2, W, 0, W * D))
    ga.close()
    gb.close()


def test_on_demand_epoch_on_a_user_stream():
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    W, D, seed = 1000, 6, 77
    g = Generator(walkers=W, seed=seed)
    s = torch.cuda.Stream()
    o = torch.empty(W * D, dtype=torch.int64, device="cuda")
    with torch.cuda.stream(s):
        o.fill_(0)
        g.epoch_begin(W, D, stream=s)
        g.consume(W, uniform=D, out=o, stream=s)
        g.epoch_end(stream=s)
        snap = o.clone()
    s.synchronize()
    got = snap.cpu().numpy().view(np.uint64).reshape(W, D)
    for t in (0, 1, 500, W - 1):
        assert np.array_equal(got[t], O.walker_draws(M32, 64, 64, seed, t, 0, D)), t
    assert g.check() == 0
    g.close()

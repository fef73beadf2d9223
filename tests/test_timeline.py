"""The Fig.4 timeline recorder (GG_TIMELINE, prng_capi.cu) and its analysis
(tools/timeline.py; §IV-A Fig.4: FEED / TRANSFER / GENERATE).
CPU: interval arithmetic.  GPU: an E-mode fill writes one interval per FEED
chunk, H2D copy and walk kernel, all inside the call's span."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import timeline as T  # noqa: E402


def test_interval_arithmetic():
    assert T.union([[5, 7], [0, 2], [1, 3], [7, 8]]) == [[0, 3], [5, 8]]
    assert T.intersect([[0, 3], [5, 8]], [[2, 6]]) == [[2, 3], [5, 6]]
    r = T.analyse([["feed", 0, 10], ["h2d", 5, 15], ["walk", 12, 20], ["walk", 25, 30]])
    assert r["span_ms"] == 0.03
    assert abs(r["gpu_idle_frac"] - (1 - 13 / 30)) < 1e-12
    assert abs(r["feed_and_h2d_frac"] - 5 / 30) < 1e-12
    assert r["feed_h2d_walk_frac"] == 0


SNIPPET = r"""
import os, sys, torch
sys.path.insert(0, %(root)r)
from paper_conf_ipps_banerjeebk12_b200 import Generator
g = Generator(walkers=4096, seed=3, epoch_draws=4)
o = torch.empty(4096 * 20, dtype=torch.int64, device="cuda")
g.fill(o)
h = torch.empty(4096 * 8, dtype=torch.int64).pin_memory()
g.fill_host(h)
torch.cuda.synchronize()
g.close()
"""


@pytest.mark.gpu
def test_timeline_records_every_stage(tmp_path):
    path = str(tmp_path / "tl.json")
    env = dict(os.environ, GG_TIMELINE=path)
    p = subprocess.run([sys.executable, "-c", SNIPPET % {"root": ROOT}], env=env,
                       capture_output=True, text=True, timeout=300)
    assert p.returncode == 0, p.stderr[-2000:]
    rows = json.load(open(path))
    kinds = {}
    for k, a, b in rows:
        assert b >= a >= -1e3, (k, a, b)  # on the handle's clock (alignment ~10 us)
        kinds[k] = kinds.get(k, 0) + 1
    # 20 draws in ring slots of 4: 5 walk kernels (+ Alg.1's feed at create);
    # fill_host: 8 draws = 2 more kernels and 2 D2H copies
    assert kinds["walk"] == 7 and kinds["d2h"] == 2
    assert kinds["feed"] >= 7 and kinds["h2d"] >= 7

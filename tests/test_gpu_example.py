"""The C/CUDA example (examples/c_consumer.cu) against the oracle: the C ABI
and the header-only prng_next used from a separately compiled user kernel,
with no Python in the data path.  Bulk fill = R11 order; on-demand = R10
(the i-th prng_next of walker t in the first epoch returns draw J0 + i,
J0 = 4 after a fill of 4 draws per walker)."""
import os
import subprocess

import pytest

import oracle as O

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
M32 = 1 << 32


@pytest.mark.parametrize("W,seed", [(1000, 0x5EED), (37, 0xABC)])
def test_c_consumer_matches_oracle(W, seed):
    exe = os.path.join(ROOT, "examples", "c_consumer")
    assert os.path.exists(exe), "build() compiles the example"
    out = subprocess.run([exe, str(W), hex(seed)[2:]], capture_output=True, text=True, timeout=120)
    assert out.returncode == 0, out.stderr
    n = 0
    for line in out.stdout.splitlines():
        kind, t, j, val = line.split()
        t, j, val = int(t), int(j), int(val, 16)
        draw = j if kind == "bulk" else 4 + j
        assert val == int(O.walker_draws(M32, 64, 64, seed, t, draw, 1)[0]), line
        n += 1
    assert n == 5 * 4 + sum(t % 3 + 1 for t in (0, 1, 2, W // 2, W - 1))


def test_python_quickstart_runs():
    import sys
    out = subprocess.run([sys.executable, os.path.join(ROOT, "examples", "quickstart.py")],
                         capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    text = out.stdout
    for key in ("bulk:", "fill_host:", "on demand:", "list ranking:", "Monte Carlo:",
                "glibc rand_r bits:", "host generator bits:"):
        assert key in text, text
    assert "tail rank 1048575" in text and "overrun flag 0" in text, text

"""The composed-step table fill kernel (GG_FILL_TABLE = warps per block,
csrc/gg_walk.cu gg_fill64t_tma_kernel) is bit-exact with the oracle for every
m = 2^k output form it serves (u64 labels of m = 2^32 with and without the
16-byte store path, u64 labels of m = 2^k < 2^32, u32 words of m <= 2^16) and
for the bipartite variant's signed table, and the any-l table kernel (l = 16,
13, 2, 101: whole and partial 4-step groups), on
ragged walker counts and fills that stop mid-draw.  The hook is read once per
process, so each configuration runs in a subprocess."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle as O

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SNIPPET = r"""
import json, sys
import numpy as np, torch
sys.path.insert(0, %(root)r)
from paper_conf_ipps_banerjeebk12_b200 import Generator
res = {}
for m, W, fmt, var, l in ((1 << 32, 1000, "u64", 0, 64), (1 << 32, 999, "u64", 0, 64),
                          (1 << 32, 4096, "u32", 0, 64), (256, 1000, "u64", 0, 64),
                          (1 << 20, 777, "u64", 0, 64), (1 << 16, 640, "u32", 0, 64),
                          (1 << 32, 1000, "u64", 1, 64), (1 << 12, 333, "u64", 1, 64),
                          (1 << 32, 1000, "u64", 0, 16), (1 << 32, 700, "u64", 0, 13),
                          (1 << 20, 500, "u64", 0, 2), (1 << 32, 300, "u64", 0, 101),
                          (1 << 16, 333, "u32", 0, 10)):
    g = Generator(walkers=W, seed=0x7AB1E + W, m=m, epoch_draws=5, variant=var, walk_len=l)
    outs = []
    for n in (7, 3 * W + 5, 2 * W + 2, 9 * W):
        if fmt == "u64":
            o = torch.empty(n, dtype=torch.int64, device="cuda")
            g.fill(o)
            outs.append(o.cpu().numpy().view(np.uint64))
        else:
            o = torch.empty(2 * n if m > 65536 else n, dtype=torch.int32, device="cuda")
            g.fill(o)
            v = o.cpu().numpy().view(np.uint32)
            outs.append(v.view(np.uint64) if m > 65536 else v.astype(np.uint64))
    g.prefetch(12)                       # resident window (K-mode) path too
    o = torch.empty(12 * W, dtype=torch.int64, device="cuda")
    g.fill(o)
    outs.append(o.cpu().numpy().view(np.uint64))
    res[f"{m}-{W}-{fmt}-{var}-{l}"] = [int(v) for v in np.concatenate(outs)]
print(json.dumps(res))
"""


@pytest.mark.parametrize("nw", ["2", "4", "8", "0"])  # 0: the R2P kernels (x2, bipartite pair)
def test_table_kernel_bit_exact(nw):
    env = dict(os.environ, GG_FILL_TABLE=nw)
    p = subprocess.run([sys.executable, "-c", SNIPPET % {"root": ROOT}], env=env,
                       capture_output=True, text=True, timeout=600)
    assert p.returncode == 0, p.stderr[-2000:]
    got = json.loads(p.stdout.strip().splitlines()[-1])
    for key, vals in got.items():
        m, W, fmt, var, l = key.split("-")
        m, W, var, l = int(m), int(W), int(var), int(l)
        total = 7 + (3 * W + 5) + (2 * W + 2) + 9 * W
        n_pref = 12 * W
        # fills continue from the running N (R11), the resident window included
        want = O.bulk_v(m, l, 64, var, 0x7AB1E + W, W, 0, total + n_pref)
        assert np.array_equal(np.array(vals, dtype=np.uint64), want), (nw, key)

"""Every diagnostic / A-B kernel and feed variant (DESIGN.md §8 hooks) is
bit-exact with the oracle: the hooks are read once per process, so each
runs in a subprocess on small C2-type inputs (ragged walker count, fills that
stop mid-draw, an on-demand epoch with a walker list, a tiny MC run)."""
import json
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle as O

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
M32 = 1 << 32

SNIPPET = r"""
import json, sys
import numpy as np, torch
sys.path.insert(0, %(root)r)
from paper_conf_ipps_banerjeebk12_b200 import Generator
W, seed = 1000, 0x5EED00F0
g = Generator(walkers=W, seed=seed, epoch_draws=3)
outs = []
for n in (7, 3 * W + 5, 2 * W):
    o = torch.empty(n, dtype=torch.int64, device="cuda")
    g.fill(o)
    outs.append(o.cpu().numpy().view(np.uint64))
bulk = np.concatenate(outs)
ids = np.arange(0, W, 7, dtype=np.uint32)
g.epoch_begin_list(ids, 2)
od = torch.empty(ids.size * 2, dtype=torch.int64, device="cuda")
g.consume(ids.size, uniform=2, out=od)
g.epoch_end()
layers = [(1.37, 1.0, 100.0, 0.9, 0.1), (1.37, 1.0, 10.0, 0.0, 0.1), (1.37, 2.0, 10.0, 0.7, 0.2)]
g2 = Generator(walkers=512, seed=0x5EED0004)
mc = g2.mc_run(layers, 2000, threads=512, epoch_draws=48)
print(json.dumps({"bulk": [int(v) for v in bulk], "od": [int(v) for v in od.cpu().numpy().view(np.uint64)],
                  "tallies": [int(v) for v in mc["tallies"]]}))
"""

# the R2P-step fill kernels run under GG_FILL_TABLE=0 (the composed-step table
# kernel is the default; tests/test_gpu_table.py covers its block sizes)
_R2P = "GG_FILL_TABLE=0 "
VARIANTS = ["GG_FILL_TABLE=0", _R2P + "GG_FILL_NO_TMA=1", _R2P + "GG_FILL_X1=1",
            _R2P + "GG_FILL_MINB=24", _R2P + "GG_FILL_STEP=0", _R2P + "GG_FILL_U2=0",
            _R2P + "GG_FILL_MINB=24 GG_FILL_U2=0",
            _R2P + "GG_FILL_ONEWAVE=1", _R2P + "GG_FILL_KPW=2", "GG_FILL_KPW=3", "GG_FILL_TABLE=2 GG_FILL_KPW=2", "GG_FILL_TABLE=8", "GG_FILL_ORB=0",
            "GG_FEED_NT_ALL=1", "GG_FEED_NO_NT=1", "GG_FEED_RATE=0", "GG_FEED_RATE=5",
            "GG_FEED_CHUNK_MB=1", "GG_FEED_CHUNKS=2", "GG_MC_MINB=4", _R2P + "GG_FILL_PAIR=1",
            "GG_FEED_STATIC=1", "GG_FEED_STATIC=1 GG_FEED_RATE=0"]


@pytest.fixture(scope="module")
def want():
    W, seed = 1000, 0x5EED00F0
    n = 7 + 3 * W + 5 + 2 * W
    bulk = O.bulk(M32, 64, 64, seed, W, 0, n)
    J0 = -(-n // W)  # first epoch starts at the next whole draw (R10)
    ids = np.arange(0, W, 7)
    lib = O.lib()
    od = []
    for t in ids:  # R10: walk the bulk draws, skip the rest of draw J0-1, then J0, J0+1
        x, y = O.walker_init(M32, 64, seed, int(t))
        xa, ya = np.array([x], np.uint64), np.array([y], np.uint64)
        for j in range((n - int(t) + W - 1) // W):
            lib.or_walker_draw(M32, 64, 64, seed, int(t), j, xa.ctypes.data, ya.ctypes.data)
        od.append([int(lib.or_walker_draw(M32, 64, 64, seed, int(t), J0 + i, xa.ctypes.data,
                                          ya.ctypes.data)) for i in range(2)])
    od = np.array(od, dtype=np.uint64)
    mc = O.mc_run(nthreads=512, photons_total=2000, D=48, seed=0x5EED0004)
    return bulk, od, mc["tallies"]


@pytest.mark.parametrize("var", VARIANTS)
def test_variant_bit_exact(var, want):
    env = dict(os.environ)
    for kv in var.split():
        k, v = kv.split("=")
        env[k] = v
    out = subprocess.run([sys.executable, "-c", SNIPPET % {"root": ROOT}], env=env,
                         capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    got = json.loads(out.stdout.strip().splitlines()[-1])
    bulk, od, tallies = want
    assert np.array_equal(np.array(got["bulk"], dtype=np.uint64), bulk), var
    # consume(): slot k's draws at [2k, 2k+1] (offsets = k * uniform)
    assert np.array_equal(np.array(got["od"], dtype=np.uint64).reshape(-1, 2), od), var
    assert got["tallies"] == [int(t) for t in tallies], var


L1_SNIPPET = r"""
import sys
import numpy as np, torch
sys.path.insert(0, %(root)r)
from paper_conf_ipps_banerjeebk12_b200 import Generator
W, seed = 32 * 700 + 5, 0x5EED00F1
g = Generator(walkers=W, seed=seed, walk_len=1)
g.prefetch(70)
o = torch.empty(W * 70 - 3, dtype=torch.int64, device="cuda")
g.fill(o)
np.save(sys.argv[1], o.cpu().numpy().view(np.uint64))
"""


@pytest.mark.parametrize("var", ["GG_FILL_KPW=2", "GG_FILL_KPW=3", "GG_FILL_ONEWAVE=1",
                                 "GG_L1_TMA_STORE=0"])
def test_l1_tma_store_several_units_per_warp(var, tmp_path):
    """l = 1 TMA-store kernel when a warp handles several 32-walker units
    (the first interior tile of a unit must not overwrite a staging
    buffer the previous unit's bulk store is still reading)."""
    env = dict(os.environ)
    k, v = var.split("=")
    env[k] = v
    f = str(tmp_path / "l1.npy")
    out = subprocess.run([sys.executable, "-c", L1_SNIPPET % {"root": ROOT}, f], env=env,
                         capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    got = np.load(f)
    W = 32 * 700 + 5
    assert np.array_equal(got, O.bulk(M32, 1, 64, 0x5EED00F1, W, 0, W * 70 - 3)), var


LR_SNIPPET = r"""
import json, sys
import numpy as np, torch
sys.path.insert(0, %(root)r)
import inputs
from paper_conf_ipps_banerjeebk12_b200 import Generator
n = 1 << 16
succ, pred, head = inputs.random_list(n, 100 + n)
g = Generator(walkers=n, seed=0x5EED0003)
rr = torch.empty(n, dtype=torch.int32, device="cuda")
sp = torch.empty(n, dtype=torch.int32, device="cuda")
rank, info = g.list_rank(torch.from_numpy(succ).cuda(), torch.from_numpy(pred).cuda(), head,
                         removed_round=rr, is_splitter=sp)
print(json.dumps({"rank": rank.cpu().tolist(), "rr": rr.cpu().tolist(), "sp": sp.cpu().tolist(),
                  "draws": info["draws"]}))
"""


@pytest.mark.parametrize("var", ["GG_LR_PREFEED=0", "GG_LR_PREFEED=2", "GG_FEED_STATIC=1",
                                 "GG_FEED_CHUNK_MB=1"])
def test_list_ranking_feed_variants_bit_exact(var):
    """List-ranking prefeed bounds (none / the survivors' lower bound / the
    default 7/8 A + 3 sd) and feed schedules give the oracle replica's FIS and
    splitter sets (2^16 nodes: every round but the last few is prefed)."""
    import inputs
    env = dict(os.environ)
    for kv in var.split():
        k, v = kv.split("=")
        env[k] = v
    out = subprocess.run([sys.executable, "-c", LR_SNIPPET % {"root": ROOT}], env=env,
                         capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr[-2000:]
    got = json.loads(out.stdout.strip().splitlines()[-1])
    n = 1 << 16
    succ, pred, head = inputs.random_list(n, 100 + n)
    want = O.lr_run(succ, pred, head, seed=0x5EED0003)
    assert np.array_equal(np.array(got["rank"], dtype=np.int32), O.lr_rank_seq(succ, head))
    assert np.array_equal(np.array(got["rr"], dtype=np.int32), want["removed_round"]), var
    assert np.array_equal(np.array(got["sp"], dtype=np.int32).astype(bool), want["is_splitter"]), var
    assert got["draws"] == want["draws"], var

"""Profile target (tool): the C4 Monte Carlo run; ncu -k regex:mc_epoch -s 3 -c 1."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_banerjeebk12_b200 import Generator  # noqa: E402

T = 1 << 20
g = Generator(walkers=T, seed=0x5EED0004)
layers = ((1.37, 1.0, 100.0, 0.9, 0.1), (1.37, 1.0, 10.0, 0.0, 0.1), (1.37, 2.0, 10.0, 0.7, 0.2))
r = g.mc_run(layers, photons_total=20 * T if len(sys.argv) < 2 else int(sys.argv[1]), threads=T)
print({k: r[k] for k in ("photons", "draws", "epochs", "kernel_us", "total_us")})

"""NIST SP 800-22 report on GPU output (tool).

    python tools/nist_report.py [out.json]
k = 100 sequences of 10^6 bits (NIST's recommended sample) of the C2
generator (m = 2^32, l = l0 = 64) computed on the GPU, in bulk order and in
walker-major order, plus the l = 1 negative control.  Per test: proportion of
sequences with P >= 0.01 (acceptance: >= 0.99 - 3 sqrt(0.0099 / k) = 0.9602)
and the uniformity P-value of the k P-values (chi-square over 10 bins,
igamc(9/2, chi2/2); acceptance >= 1e-4), as in SP 800-22 §4.2.
"""
import json
import math
import os
import sys
from multiprocessing import get_context

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
from scipy import special  # noqa: E402

K, NBITS = int(os.environ.get("NIST_K", "100")), 1_000_000


def _one(bits):
    import nist as N
    return N.run(bits)


def summarize(results):
    out = {}
    k = len(results)
    bound = 0.99 - 3 * math.sqrt(0.99 * 0.01 / k)
    for name in results[0]:
        p = np.array([r[name] for r in results])
        prop = float((p >= 0.01).mean())
        cnt = np.histogram(p, bins=10, range=(0, 1))[0]
        chi2 = float(((cnt - k / 10) ** 2 / (k / 10)).sum())
        unif = float(special.gammaincc(4.5, chi2 / 2))
        out[name] = {"proportion": prop, "uniformity_p": unif,
                     "pass": bool(prop >= bound and unif >= 1e-4)}
    return out, bound


def sequences(z):
    import nist as N
    bits = N.bits_of_words(np.ascontiguousarray(z).reshape(-1).view(np.uint32))
    return [bits[i * NBITS:(i + 1) * NBITS].copy() for i in range(K)]


def main():
    import torch
    from paper_conf_ipps_banerjeebk12_b200 import Generator
    report = {"k": K, "bits_per_sequence": NBITS}
    runs = {}
    for l, label in ((64, "l64"), (1, "l1_negative_control")):
        W = 1 << 16 if l == 64 else 1 << 10
        D = -(-K * NBITS // (64 * W))  # draws so that W * D labels hold K sequences
        g = Generator(walkers=W, seed=0x5EED0002, walk_len=l)
        o = torch.empty(W * D, dtype=torch.int64, device="cuda")
        g.fill(o)
        torch.cuda.synchronize()
        z = o.view(D, W).cpu().numpy()
        g.close()
        if l == 64:
            runs[f"{label}_bulk"] = sequences(z)
        runs[f"{label}_walker_major"] = sequences(z.T.copy())
    with get_context("spawn").Pool(os.cpu_count() or 1) as pool:
        for name, seqs in runs.items():
            res, bound = summarize(pool.map(_one, seqs))
            report[name] = res
            report["proportion_bound"] = bound
            print(name, {k: (round(v["proportion"], 2), round(v["uniformity_p"], 4), v["pass"])
                         for k, v in res.items()}, file=sys.stderr)
    out = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out", "nist.json")
    with open(out, "w") as f:
        json.dump(report, f, indent=1)


if __name__ == "__main__":
    main()

"""Build the native library libggprng.so in-tree (sm_100a only).

    python paper_conf_ipps_banerjeebk12_b200/build.py [--force]

nvcc cross-compiles for sm_100a without a GPU; the .so travels to the GPU
box with the repo snapshot.  CUDA runtime is linked statically so the
library does not depend on which libcudart torch loaded.
"""
from __future__ import annotations

import os
import subprocess
import sys

PKG = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(PKG)
CSRC = os.path.join(PKG, "csrc")
INCLUDE = os.path.join(ROOT, "include")
LIB = os.path.join(PKG, "libggprng.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CUDA_FLAGS = ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-O2",
                     "-Xptxas", "-O3", "--expt-relaxed-constexpr"]
CXX_FLAGS = ["-O3", "-fPIC", "-std=c++17", "-fno-fast-math"]
# mc.cu: fp64 physics evaluated exactly as written (no FMA contraction), to
# match the CPU oracle expression by expression.
PER_FILE_FLAGS = {"mc.cu": ["-fmad=false"]}


def sources():
    cu = sorted(f for f in os.listdir(CSRC) if f.endswith(".cu"))
    cpp = sorted(f for f in os.listdir(CSRC) if f.endswith(".cpp"))
    return [os.path.join(CSRC, f) for f in cu], [os.path.join(CSRC, f) for f in cpp]


def _deps():
    cu, cpp = sources()
    hdrs = [os.path.join(CSRC, f) for f in os.listdir(CSRC) if f.endswith((".h", ".cuh"))]
    hdrs += [os.path.join(INCLUDE, f) for f in os.listdir(INCLUDE)]
    return cu + cpp + hdrs + [os.path.abspath(__file__)]


def up_to_date() -> bool:
    if not os.path.exists(LIB):
        return False
    t = os.path.getmtime(LIB)
    return all(os.path.getmtime(d) <= t for d in _deps())


def build(force: bool = False, verbose: bool = False) -> str:
    if not force and up_to_date():
        return LIB
    cu, cpp = sources()
    objdir = os.path.join(PKG, "build")
    os.makedirs(objdir, exist_ok=True)
    objs = []
    procs = []
    for src in cu:
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        extra = PER_FILE_FLAGS.get(os.path.basename(src), [])
        cmd = [NVCC] + CUDA_FLAGS + extra + ["-I", INCLUDE, "-I", CSRC, "-c", src, "-o", obj]
        procs.append((cmd, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)))
        objs.append(obj)
    for src in cpp:
        obj = os.path.join(objdir, os.path.basename(src) + ".o")
        cmd = ["g++"] + CXX_FLAGS + ["-I", INCLUDE, "-I", CSRC, "-I", "/usr/local/cuda/include",
                                     "-c", src, "-o", obj]
        procs.append((cmd, subprocess.Popen(cmd, stdout=subprocess.PIPE, stderr=subprocess.STDOUT)))
        objs.append(obj)
    failed = False
    for cmd, p in procs:
        out, _ = p.communicate()
        if verbose or p.returncode != 0:
            sys.stderr.write(" ".join(cmd) + "\n" + out.decode(errors="replace"))
        failed |= p.returncode != 0
    if failed:
        raise RuntimeError("libggprng build failed")
    tmp = LIB + f".tmp{os.getpid()}"
    cmd = [NVCC] + ARCH + ["-shared", "-Xcompiler", "-fPIC", "-o", tmp] + objs + \
        ["-lpthread", "-cudart", "static"]
    subprocess.check_call(cmd)
    os.replace(tmp, LIB)
    build_examples()
    return LIB


EXAMPLES = os.path.join(ROOT, "examples")


def build_examples() -> None:
    """C/CUDA programs that use only include/ and libggprng.so (no Python)."""
    if not os.path.isdir(EXAMPLES):
        return
    for f in sorted(os.listdir(EXAMPLES)):
        if not f.endswith(".cu"):
            continue
        exe = os.path.join(EXAMPLES, f[:-3])
        cmd = [NVCC] + ARCH + ["-O2", "-std=c++17", "-I", INCLUDE, os.path.join(EXAMPLES, f),
                               "-o", exe, "-L", PKG, "-lggprng", "-Xlinker",
                               "-rpath,$ORIGIN/../" + os.path.basename(PKG)]
        subprocess.check_call(cmd)


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose="-v" in sys.argv)
    print(LIB)

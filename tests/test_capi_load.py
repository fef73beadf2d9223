"""The C-ABI library loads and exports every symbol include/*.h declares (no GPU)."""
import ctypes
import os
import re
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
INCLUDE = os.path.join(ROOT, "include")


def declared_functions():
    names = set()
    for f in os.listdir(INCLUDE):
        if not f.endswith(".h"):
            continue
        src = open(os.path.join(INCLUDE, f)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        for m in re.finditer(r"^(?:int|const char \*|void)\s*\*?\s*(\w+)\s*\(", src, flags=re.M):
            names.add(m.group(1))
    return sorted(names)


@pytest.fixture(scope="module")
def lib():
    from paper_conf_ipps_banerjeebk12_b200 import _lib
    return _lib


def test_headers_declare_the_boundary():
    names = declared_functions()
    for must in ("prng_create", "prng_fill", "prng_fill_host", "prng_prefetch", "prng_epoch_begin",
                 "prng_epoch_end", "prng_device_view", "prng_check", "prng_destroy",
                 "gg_consume"):
        assert must in names


def test_every_declared_symbol_is_exported(lib):
    so = lib.LIB_PATH
    out = subprocess.check_output(["nm", "-D", "--defined-only", so]).decode()
    exported = set(line.split()[-1] for line in out.splitlines() if " T " in line)
    missing = [n for n in declared_functions() if n not in exported]
    assert not missing, missing
    # and the Python binding binds exactly the same names
    assert set(lib.EXPORTED) == set(declared_functions())


def test_so_is_sm100a(lib):
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "-lelf", lib.LIB_PATH]).decode()
    assert "sm_100a" in out


def test_host_only_calls(lib):
    assert lib.prng_version() >= 100
    assert lib.prng_strerror(lib.PRNG_E_OVERRUN).decode().startswith("on-demand")
    p = lib.prng_graph_params()
    assert lib.prng_default_params(ctypes.byref(p)) == 0
    assert (p.m, p.degree, p.walk_len, p.burnin_len) == (1 << 32, 7, 64, 64)
    # invalid arguments are rejected before any device work
    h = ctypes.c_void_p()
    assert lib.prng_create(ctypes.byref(h), None, 16, 0, None) == lib.PRNG_E_INVALID
    p.degree = 5
    assert lib.prng_create(ctypes.byref(h), ctypes.byref(p), 16, 0, None) == lib.PRNG_E_UNSUPPORTED
    p.degree = 7
    p.m = (1 << 32) + 1  # beyond the 64-bit label space (m^2 <= 2^64)
    assert lib.prng_create(ctypes.byref(h), ctypes.byref(p), 16, 0, None) == lib.PRNG_E_INVALID
    p.m = 1
    assert lib.prng_create(ctypes.byref(h), ctypes.byref(p), 16, 0, None) == lib.PRNG_E_INVALID
    p.m = 1 << 32
    assert lib.prng_create(ctypes.byref(h), ctypes.byref(p), 0, 0, None) == lib.PRNG_E_INVALID
    assert lib.prng_create(ctypes.byref(h), ctypes.byref(p), (1 << 24) + 1, 0, None) == lib.PRNG_E_INVALID
    o = lib.prng_options()
    assert lib.prng_default_options(ctypes.byref(o)) == 0
    o.bit_source = 4  # PRNG_BITS_* ends at PRNG_BITS_GGCPU = 3
    assert lib.prng_create(ctypes.byref(h), ctypes.byref(p), 16, 0, ctypes.byref(o)) == lib.PRNG_E_INVALID
    o.bit_source = 2  # callback without a function
    assert lib.prng_create(ctypes.byref(h), ctypes.byref(p), 16, 0, ctypes.byref(o)) == lib.PRNG_E_INVALID
    assert not h.value  # nothing was created
    assert lib.prng_destroy(None) == 0
    assert lib.prng_fill(None, None, 1, 0, None) == lib.PRNG_E_INVALID


def test_product_package_does_not_touch_oracle():
    # the product path never imports, includes, links or loads anything under oracle/
    pat = re.compile(r"import\s+oracle|from\s+oracle|oracle/|libggoracle|or_[a-z_]+\(|#include\s+\"[^\"]*oracle")
    for d in ("paper_conf_ipps_banerjeebk12_b200", "include"):
        for dp, _, fs in os.walk(os.path.join(ROOT, d)):
            for f in fs:
                if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                    src = open(os.path.join(dp, f)).read()
                    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)   # C comments
                    src = re.sub(r"(//|#(?!include)).*", "", src)       # line comments
                    assert not pat.search(src), (f, pat.search(src))

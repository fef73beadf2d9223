"""Diagnostic (tool): H2D copy rates from the library's pinned chunks (gg_debug_h2d_probe)."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_banerjeebk12_b200 import Generator, _lib  # noqa: E402

g = Generator(walkers=1024, seed=1)
fn = _lib.lib().gg_debug_h2d_probe
fn.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
fn(g.handle, 24 << 20)

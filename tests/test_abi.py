"""The C-ABI library loads on a GPU-less host and exports every symbol the
headers declare; host-side calls behave (CPU only, no compute calls)."""
import ctypes
import glob
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    names = set()
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        src = open(h).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        for m in re.finditer(r"^\s*(?:const\s+char\s*\*|int32_t|int|void)\s*\*?\s*(arlo_\w+)\s*\(", src, re.M):
            names.add(m.group(1))
    return names


def test_headers_declare_the_boundary():
    names = declared_symbols()
    for required in ("arlo_runtime_create", "arlo_infer", "arlo_allocate", "arlo_dispatch",
                     "arlo_weights_create", "arlo_op_gemm", "arlo_op_attention"):
        assert required in names


def test_library_exports_every_declared_symbol(arlo_lib):
    lib = ctypes.CDLL(arlo_lib.LIB_PATH)
    missing = [n for n in declared_symbols() if not hasattr(lib, n)]
    assert not missing, missing
    assert set(arlo_lib.EXPORTED) == declared_symbols()


def test_version_and_error_strings(arlo_lib):
    assert "sm_100a" in arlo_lib.version()
    assert arlo_lib.lib.arlo_last_error() is not None


def test_weights_create_rejects_bad_config_without_gpu(arlo_lib):
    from paper_conf_icpp_tanlyl024_b200 import workload as wl
    c = arlo_lib.make_config(wl.TINY, arlo_lib.BF16)
    c.hidden = 100  # not 64 * heads
    h = ctypes.c_void_p()
    arr = (ctypes.c_void_p * 1)()
    rc = arlo_lib.lib.arlo_weights_create(0, ctypes.byref(c), arr, 1, ctypes.byref(h))
    assert rc == arlo_lib.EINVAL
    assert "64" in arlo_lib.lib.arlo_last_error().decode()
    c2 = arlo_lib.make_config(wl.TINY, arlo_lib.BF16)
    assert arlo_lib.lib.arlo_weights_count(ctypes.byref(c2)) == 5 + 12 * 2 + 4


@pytest.mark.skipif(__import__("torch").cuda.is_available(), reason="CPU-only behaviour")
def test_no_device_is_reported(arlo_lib):
    from paper_conf_icpp_tanlyl024_b200 import workload as wl
    c = arlo_lib.make_config(wl.TINY, arlo_lib.BF16)
    n = arlo_lib.lib.arlo_weights_count(ctypes.byref(c))
    bufs = [np.zeros(8, np.float32) for _ in range(n)]
    arr = (ctypes.c_void_p * n)(*[b.ctypes.data for b in bufs])
    h = ctypes.c_void_p()
    rc = arlo_lib.lib.arlo_weights_create(0, ctypes.byref(c), arr, n, ctypes.byref(h))
    assert rc in (arlo_lib.ENODEV, arlo_lib.EINVAL)

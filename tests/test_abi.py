"""C-ABI checks that need no GPU: the library loads, exports every function
include/gala.h declares, and its host-only helpers behave."""
import ctypes
import subprocess

import numpy as np
import pytest

import paper_conf_ppopp_wangllwm00z25_b200 as gala


def test_library_exports_every_declared_symbol():
    L = gala.lib()
    names = gala.declared_functions()
    assert len(names) >= 15
    missing = [f for f in names if not hasattr(L, f)]
    assert not missing, missing


def test_exported_symbols_are_extern_c():
    out = subprocess.check_output(["nm", "-D", "--defined-only", gala.LIB_PATH], text=True)
    syms = {line.split()[-1] for line in out.splitlines() if line.strip()}
    for f in gala.declared_functions():
        assert f in syms, f


def test_library_is_sm100a():
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", gala.LIB_PATH], text=True)
    assert "sm_100a" in out


def test_version_and_null_handle_errors():
    assert "sm_100a" in gala.version()
    L = gala.lib()
    assert L.gala_set_option(None, b"prune", 1) == 1
    assert L.gala_run(None, 1.0, 1e-6, 0) == 1
    assert "null" in L.gala_last_error().decode()
    q = ctypes.c_double()
    assert L.gala_modularity(None, ctypes.byref(q)) == 1


def test_partition_ranges_edge_balanced():
    rng = np.random.default_rng(0)
    deg = rng.integers(0, 50, size=1000)
    rp = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
    for world in (1, 2, 4, 8):
        b = gala.partition_ranges(rp, world)
        assert b[0] == 0 and b[-1] == 1000 and np.all(np.diff(b) >= 0)
        loads = rp[b[1:]] - rp[b[:-1]]
        assert loads.max() - loads.min() <= 2 * deg.max() + 1


def test_header_has_no_torch_types():
    import re
    src = re.sub(r"/\*.*?\*/", "", open(gala.HEADER_PATH).read(), flags=re.S)
    for bad in ("torch", "at::", "Tensor", "std::"):
        assert bad not in src

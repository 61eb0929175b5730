"""CPU checks of the boundary: the C-ABI library loads and exports every symbol
include/gallatin.h declares; the oracle builds; nothing computes without a GPU."""
import ctypes
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def built():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ppopp_mccoyp24_b200 as G
    return G


def test_library_exports_every_declared_symbol(built):
    G = built
    names = G.declared_functions()
    assert len(names) >= 30
    L = ctypes.CDLL(G._native.LIB_PATH)
    missing = [n for n in names if not hasattr(L, n)]
    assert not missing, missing


def test_library_is_sm100a(built):
    out = subprocess.run(["cuobjdump", "--list-elf", built._native.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_oracle_and_product_share_no_code():
    """The oracle never includes the CUDA headers and the product never imports the oracle."""
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".c", ".py", ".h")):
            lines = open(os.path.join(ROOT, "oracle", f)).read().splitlines()
            code = [ln for ln in lines if ln.lstrip().startswith(("#include", "import ", "from "))]
            assert not any("gallatin" in ln or "paper_conf" in ln for ln in code), f
    pkg = os.path.join(ROOT, "paper_conf_ppopp_mccoyp24_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                text = open(os.path.join(dp, f)).read()
                assert "import oracle" not in text and "from oracle" not in text and "oracle/" not in text, f


def test_error_paths_without_gpu(built):
    G = built
    L = G.lib()
    assert L.gallatin_is_initialized() == 0
    assert L.gallatin_destroy() == G._native.ERR_STATE
    assert L.gallatin_malloc(None, None, 5, None) == G._native.ERR_STATE
    assert L.gallatin_error_string(-1) == b"invalid argument"
    assert L.veb_create(0, ctypes.byref(ctypes.c_void_p())) == G._native.ERR_INVALID
    assert L.veb_create(33, ctypes.byref(ctypes.c_void_p())) == G._native.ERR_INVALID

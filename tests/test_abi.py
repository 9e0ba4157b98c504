"""CPU-side checks of the C-ABI library: it builds for sm_100a, loads, and
exports every symbol include/tg.h declares (no compute calls without a GPU)."""
import ctypes
import os
import re
import subprocess

import pytest

from tests.conftest import ROOT


def _declared():
    hdr = open(os.path.join(ROOT, "include", "tg.h")).read()
    hdr = re.sub(r"/\*.*?\*/", "", hdr, flags=re.S)
    return sorted(set(re.findall(r"\b(tg_[a-z_]+)\s*\(", hdr)))


@pytest.fixture(scope="module")
def libpath():
    from paper_conf_ppopp_wangm23_b200.build import build
    return build()


def test_header_declares_the_boundary():
    names = _declared()
    for f in ("tg_graph_load", "tg_model_load", "tg_embed_batch", "tg_score_edges", "tg_cache_reset"):
        assert f in names


def test_library_exports_every_declared_symbol(libpath):
    out = subprocess.run(["nm", "-D", "--defined-only", libpath], capture_output=True, text=True).stdout
    exported = set(re.findall(r" T (tg_\w+)", out))
    missing = [n for n in _declared() if n not in exported]
    assert not missing, missing


def test_library_loads_and_reports_version(libpath):
    L = ctypes.CDLL(libpath)
    L.tg_version.restype = ctypes.c_char_p
    assert b"sm_100a" in L.tg_version()
    L.tg_strerror.restype = ctypes.c_char_p
    assert L.tg_strerror(-1) == b"invalid argument"


def test_binding_exports_match_header():
    from paper_conf_ppopp_wangm23_b200 import tg
    assert set(tg.EXPORTS) == set(_declared())


def test_cubin_is_sm100a_with_no_fallback(libpath):
    out = subprocess.run(["cuobjdump", "--list-elf", libpath], capture_output=True, text=True).stdout
    assert "sm_100a" in out
    # the product path never imports the oracle
    pkg = os.path.join(ROOT, "paper_conf_ppopp_wangm23_b200")
    for f in os.listdir(pkg):
        if f.endswith(".py"):
            src = open(os.path.join(pkg, f)).read()
            assert "import oracle" not in src and "from oracle" not in src, f


def test_null_and_invalid_args_rejected_without_gpu(libpath):
    L = ctypes.CDLL(libpath)
    L.tg_graph_load.argtypes = [ctypes.c_int, ctypes.c_void_p, ctypes.c_void_p]
    assert L.tg_graph_load(0, None, None) == -1
    L.tg_cache_reset.argtypes = [ctypes.c_void_p, ctypes.c_int64]
    assert L.tg_cache_reset(None, -1) == -1
    L.tg_kernel_launches.argtypes = [ctypes.c_void_p]
    L.tg_kernel_launches.restype = ctypes.c_int64
    assert L.tg_kernel_launches(None) == 0

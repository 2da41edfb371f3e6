"""C-ABI library checks that need no GPU (-m "not gpu"): it loads, it exports every
entry point include/gp.h declares, and the product path refuses to run without a device."""
import ctypes
import os
import re
import subprocess

import pytest
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def gp():
    from paper_conf_ipps_goodarzibg16_b200 import _build
    _build.build()
    import paper_conf_ipps_goodarzibg16_b200.gp as gp
    return gp


def test_header_declares_the_north_star_calls(gp):
    syms = gp.exported_symbols()
    for name in ("gp_graph_create", "gp_match_level", "gp_contract_level", "gp_coarsen_to", "gp_free"):
        assert name in syms


def test_library_exports_every_declared_symbol(gp):
    lib = ctypes.CDLL(gp.LIB)
    missing = [s for s in gp.exported_symbols() if not hasattr(lib, s)]
    assert not missing, missing


def test_only_abi_symbols_are_exported(gp):
    out = subprocess.run(["nm", "-D", "--defined-only", gp.LIB], capture_output=True, text=True).stdout
    names = [l.split()[-1] for l in out.splitlines() if " T " in l]
    assert names and all(n.startswith("gp_") for n in names), names
    assert sorted(names) == sorted(gp.exported_symbols())


def test_library_is_sm100a_only(gp):
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", gp.LIB], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out
    assert re.findall(r"sm_\d+a?", out) and set(re.findall(r"sm_\d+a?", out)) == {"sm_100a"}


def test_status_strings(gp):
    for code, name in gp.STATUS.items():
        assert gp._lib.gp_status_string(code).decode() == name


def test_invalid_handles_are_rejected(gp):
    assert gp._lib.gp_match_level(None, None, 0, None) == 1
    assert gp._lib.gp_coarsen_to(None, None, None) == 1
    gp._lib.gp_free(None)  # NULL-safe


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU behaviour")
def test_no_cpu_fallback(gp):
    with pytest.raises(RuntimeError):
        gp.Context(0)
    h = ctypes.c_void_p()
    st = gp._lib.gp_ctx_create(0, None, ctypes.byref(h))
    assert st != 0 and not h.value

"""The C-ABI library loads and exports every entry point include/stg.h declares
(-m "not gpu": no compute calls, no device needed)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "stg.h")


def _declared_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"\b(stg_[a-z0-9_]+)\s*\(", src)
    return sorted(set(n for n in names if not n.endswith("_fn")))


def test_header_declares_the_north_star_calls():
    names = _declared_functions()
    for n in ("stg_static_graph_create", "stg_dtdg_create", "stg_dtdg_get_snapshot",
              "stg_gcn_aggregate_fwd", "stg_gcn_aggregate_bwd", "stg_tgcn_step"):
        assert n in names


def test_library_exports_every_declared_symbol(stg):
    lib = ctypes.CDLL(stg.LIB_PATH)
    missing = [n for n in _declared_functions() if not hasattr(lib, n)]
    assert not missing, missing
    assert set(stg.ABI_SYMBOLS) <= set(_declared_functions())


def test_library_is_sm100a_only(stg):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", stg.LIB_PATH],
                         capture_output=True, text=True).stdout
    archs = set(re.findall(r"sm_(\d+a?)", out))
    assert archs == {"100a"}, archs


def test_no_oracle_in_product_path():
    """The product package never imports or links the oracle."""
    pkg = os.path.join(ROOT, "paper_conf_ipps_cherianmcc24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f), errors="replace").read()
                assert "import oracle" not in txt and "from oracle" not in txt, f
                assert "stg_oracle" not in txt and "liboracle" not in txt, f


def test_errors_are_reported_without_a_device(stg):
    """Argument validation is synchronous and needs no GPU."""
    v = stg.stg_csr_view()
    with pytest.raises(stg.StgError) as e:
        stg._check(stg._lib.stg_gcn_aggregate_fwd(ctypes.byref(v), 0, None, 0, None, 0, None))
    assert e.value.status == 1
    h = ctypes.c_void_p()
    st = stg._lib.stg_static_graph_create(0, 0, None, None, 0, None, None, ctypes.byref(h))
    assert st == 2 and b"V=0" in stg._lib.stg_last_error()
    assert stg._lib.stg_dtdg_num_edges(None, 0) == -1

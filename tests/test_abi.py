"""The C-ABI library loads and exports every entry point include/wg.h declares
(no compute calls: this runs without a GPU)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "wg.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:wg_status|const char\*|int64_t|size_t)\s+(wg_\w+)\s*\(", src, flags=re.M)))


def test_header_declares_the_boundary():
    names = declared_symbols()
    for must in ("wg_graph_create", "wg_plan_create", "wg_conv_forward", "wg_conv_backward"):
        assert must in names


def test_library_exports_every_declared_symbol():
    from paper_conf_eurosys_huangz0wjzzzys24_b200 import _capi
    if not os.path.exists(_capi.LIB_PATH):
        import __graft_entry__
        __graft_entry__.build()
    lib = ctypes.CDLL(_capi.LIB_PATH)
    for name in declared_symbols():
        assert hasattr(lib, name), name
    assert sorted(_capi.EXPORTS) == declared_symbols()


def test_status_strings_without_gpu():
    from paper_conf_eurosys_huangz0wjzzzys24_b200 import _capi
    L = _capi.lib()
    assert L.wg_status_string(0) == b"ok"
    assert L.wg_status_string(6) == b"unsupported"


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_eurosys_huangz0wjzzzys24_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in txt and "from oracle" not in txt and "wg_oracle" not in txt, f

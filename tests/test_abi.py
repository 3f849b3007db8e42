"""C-ABI contract checks that need no GPU: the library loads and exports every
symbol include/tg.h declares; status strings; the binding refuses to fall back."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "tg.h")


@pytest.fixture(scope="module")
def lib():
    from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import _build
    _build.build()
    from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph
    return tempgraph.load_library()


def declared_symbols():
    text = open(HEADER).read()
    return sorted(set(re.findall(r"TG_API\s+[\w\s\*]+?\b(tg_\w+)\s*\(", text)))


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for s in ("tg_graph_create", "tg_build_chains", "tg_query", "tg_graph_destroy", "tg_last_error"):
        assert s in syms


def test_every_declared_symbol_is_exported(lib):
    for s in declared_symbols():
        assert hasattr(lib, s), s
        getattr(lib, s)  # resolves through dlsym


def test_binding_names_match_header():
    from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph
    assert sorted(tempgraph.EXPORTED) == declared_symbols()


def test_status_strings(lib):
    for i, name in enumerate(["TG_OK", "TG_ERR_INVALID", "TG_ERR_RANGE", "TG_ERR_NOMEM", "TG_ERR_CUDA",
                              "TG_ERR_STATE", "TG_ERR_NCCL"]):
        assert lib.tg_status_string(i).decode() == name


def test_create_argument_errors_without_gpu(lib):
    """Argument checks happen before any device work."""
    h = ctypes.c_void_p()
    assert lib.tg_graph_create(0, 0, None, None, None, None, None, 0, ctypes.byref(h)) == 1  # n = 0
    assert lib.tg_graph_create(4, 3, None, None, None, None, None, 0, ctypes.byref(h)) == 1  # NULL arrays
    assert lib.tg_graph_create(4, 0, None, None, None, None, None, 0, None) == 1            # NULL out
    assert lib.tg_build_chains(None) == 1
    lib.tg_graph_destroy(None)  # NULL-safe


def test_create_without_device_reports_cuda_error(lib):
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    h = ctypes.c_void_p()
    assert lib.tg_graph_create(4, 0, None, None, None, None, None, 0, ctypes.byref(h)) == 4
    assert b"CUDA" in lib.tg_last_error() or b"device" in lib.tg_last_error()


def test_no_silent_fallback(tmp_path):
    from paper_conf_asplos_0003wh0dhwy0lyl25_b200 import tempgraph
    with pytest.raises(RuntimeError):
        tempgraph._lib_saved = tempgraph._lib
        tempgraph._lib = None
        try:
            tempgraph.load_library(str(tmp_path / "missing.so"))
        finally:
            tempgraph._lib = tempgraph._lib_saved


def test_product_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_asplos_0003wh0dhwy0lyl25_b200")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                src = open(os.path.join(dp, f)).read()
                assert "oracle" not in re.sub(r"(?m)^\s*(//|#).*$", "", src).replace("Nothing here is shared with oracle", ""), f

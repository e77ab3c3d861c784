"""The C-ABI library loads and exports every symbol include/sbr.h declares (CPU only).

No compute calls here (no GPU in this environment); only host-side logic that
does not touch a device: status strings, version, workspace sizing.
"""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "sbr.h")


def declared_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(sbr_[a-z_0-9]+)\s*\(", text)))


@pytest.fixture(scope="module")
def lib():
    import __graft_entry__

    __graft_entry__.build()
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    return _lib.lib()


def test_header_declares_the_boundary():
    fns = declared_functions()
    for name in ["sbr_create", "sbr_destroy", "sbr_workspace_query", "sbr_reduce", "sbr_reduce_host",
                 "sbr_status_string", "sbr_generate_symmetric", "sbr_kernel_stats"]:
        assert name in fns


def test_every_declared_symbol_is_exported(lib):
    from paper_conf_ppopp_zhangsoyw23_b200 import _lib

    for name in declared_functions():
        assert hasattr(lib, name), f"{name} declared in sbr.h but not exported"
        assert name in _lib.SIGNATURES, f"{name} has no ctypes signature in the binding"


def test_no_torch_types_in_the_abi():
    code = re.sub(r"/\*.*?\*/", "", open(HEADER).read(), flags=re.S)
    assert "torch" not in code and "at::" not in code and "Tensor" not in code


def test_status_strings_and_version(lib):
    assert lib.sbr_status_string(0) == b"ok"
    assert b"Inf" in lib.sbr_status_string(1)
    assert b"argument 4" in lib.sbr_status_string(-4)
    assert lib.sbr_version().startswith(b"libsbr")


def test_workspace_query_and_argument_errors(lib):
    out = ctypes.c_size_t()
    assert lib.sbr_workspace_query(None, 256, 8, 32, 0, ctypes.byref(out)) == 0
    small = out.value
    assert small > 0
    assert lib.sbr_workspace_query(None, 4096, 32, 256, 0, ctypes.byref(out)) == 0
    assert out.value > small
    assert lib.sbr_workspace_query(None, 0, 8, 32, 0, ctypes.byref(out)) == -2
    assert lib.sbr_workspace_query(None, 256, 0, 32, 0, ctypes.byref(out)) == -3
    assert lib.sbr_workspace_query(None, 256, 8, 12, 0, ctypes.byref(out)) == -4
    assert lib.sbr_workspace_query(None, 256, 8, 32, 7, ctypes.byref(out)) == -5
    assert lib.sbr_workspace_query(None, 8, 8, 32, 0, ctypes.byref(out)) == 0 and out.value == 0
    # a NULL handle is argument 1 for the compute entry points
    assert lib.sbr_reduce(None, 0, 16, 4, 8, None, 16, None, 5, None, 16) == -1
    assert lib.sbr_launch_count(None) == -1


def test_product_path_has_no_oracle_or_cpu_fallback():
    """The package must not import the oracle or fall back to CPU math."""
    pkg = os.path.join(ROOT, "paper_conf_ppopp_zhangsoyw23_b200")
    for fn in os.listdir(pkg):
        if fn.endswith(".py"):
            src = open(os.path.join(pkg, fn)).read()
            assert "oracle" not in src.replace("no oracle", ""), fn
            assert "numpy.linalg" not in src and "np.linalg" not in src, fn
            assert "torch.linalg" not in src, fn

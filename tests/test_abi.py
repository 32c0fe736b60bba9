"""The C-ABI boundary without a GPU: the library builds, loads, exports every symbol that
include/tbc.h declares, and fails loudly (status codes, no crash) when no device exists."""
import ctypes
import os
import re

import numpy as np
import pytest

import paper_conf_icppw_artiless21_b200 as tbc

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    text = open(os.path.join(ROOT, "include", "tbc.h")).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"\b(tbc_[a-z_]+)\s*\(", text)))


def test_header_and_binding_agree():
    assert declared_symbols() == sorted(tbc.SYMBOLS)


def test_library_exports_every_declared_symbol():
    L = tbc.lib()
    for name in declared_symbols():
        assert hasattr(L, name), name


def test_library_is_sm100a():
    path = tbc.lib()._name
    out = os.popen(f"cuobjdump --list-elf {path} 2>&1").read()
    assert "sm_100a" in out, out


def test_status_strings():
    L = tbc.lib()
    assert L.tbc_status_string(0) == b"TBC_OK"
    assert L.tbc_status_string(1) == b"TBC_ERR_INVALID"
    assert L.tbc_status_string(4) == b"TBC_ERR_UNSUPPORTED"


def test_invalid_arguments_rejected_before_touching_a_device():
    cp = np.array([0, 1, 2], dtype=np.int64)
    ri = np.array([1, 0], dtype=np.int32)
    with pytest.raises(tbc.TBCError) as e:
        tbc.Graph.from_csc(np.array([1, 1, 2], dtype=np.int64), ri, directed=False)
    assert e.value.status == 1
    with pytest.raises(tbc.TBCError) as e:
        tbc.Graph.from_csc(cp, np.array([1, 5], dtype=np.int32), directed=False)
    assert e.value.status == 1
    with pytest.raises(tbc.TBCError) as e:
        tbc.Graph.from_coo(3, [0, 1], [1, 7], directed=True)
    assert e.value.status == 1
    L = tbc.lib()
    assert L.tbc_destroy(None) == 0


def test_no_gpu_means_an_error_not_a_fallback():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    cp = np.array([0, 1, 2], dtype=np.int64)
    ri = np.array([1, 0], dtype=np.int32)
    with pytest.raises(tbc.TBCError) as e:
        tbc.Graph.from_csc(cp, ri, directed=False)
    assert e.value.status in (1, 3)

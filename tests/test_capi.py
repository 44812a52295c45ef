"""C-ABI checks that need no GPU: the library loads, exports every function include/sassi.h
declares, the host-only layout call agrees with the oracle's independent layout, and without a
CUDA device the product fails loudly (no CPU fallback)."""
import ctypes
import os
import re

import numpy as np
import pytest

import oracle
from paper_conf_isca_stephensonhlejn15_b200 import sassi

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    names = set()
    for h in sorted(os.listdir(os.path.join(ROOT, "include"))):
        if h.endswith(".h"):
            src = open(os.path.join(ROOT, "include", h)).read()
            src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
            names |= set(re.findall(r"\b(sassi_[a-z0-9_]+)\s*\(", src))
    return sorted(names)


def test_header_declares_the_north_star_entry_points():
    names = declared_functions()
    for n in ("sassi_ctx_create", "sassi_attach_handler", "sassi_consume", "sassi_read_tables",
              "sassi_merge", "sassi_sample_sites", "sassi_reset", "sassi_strerror"):
        assert n in names


def test_library_exports_every_declared_symbol():
    L = ctypes.CDLL(sassi.LIB_PATH)
    missing = [n for n in declared_functions() if not hasattr(L, n)]
    assert not missing, missing
    # and the binding wraps each of them under the same name
    assert set(declared_functions()) == set(sassi.SIGNATURES)
    for n in declared_functions():
        assert callable(getattr(sassi, n))


@pytest.mark.parametrize("S,W", [(0, 0), (1, 1), (7, 2), (204, 131072), (4096, 3)])
def test_layout_agrees_with_oracle(S, W):
    assert sassi.sassi_table_layout(S, W) == oracle.layout(S, W) | {"diag": 0}


def test_strerror_names_every_status():
    for st in range(0, -8, -1):
        assert sassi.sassi_strerror(st) != "unknown status"


def _has_gpu():
    try:
        import torch
        return torch.cuda.is_available()
    except Exception:
        return False


@pytest.mark.skipif(_has_gpu(), reason="checks the no-GPU behaviour")
def test_no_cpu_fallback_without_gpu():
    s = np.zeros(1, dtype=sassi.SITE_DTYPE)
    s[0]["pc"] = 0x10
    with pytest.raises(sassi.SassiError) as e:
        sassi.sassi_ctx_create(0, s, 1)
    assert e.value.status == sassi.SASSI_ECUDA


def test_site_validation_precedes_device_use():
    s = np.zeros(2, dtype=sassi.SITE_DTYPE)
    s["pc"] = [0x10, 0x10]                       # duplicate pc
    with pytest.raises(sassi.SassiError) as e:
        sassi.sassi_ctx_create(0, s, 1)
    assert e.value.status == sassi.SASSI_EINVAL
    s["pc"] = [0x10, 0xFFFFFFFF]                 # reserved pc
    with pytest.raises(sassi.SassiError) as e:
        sassi.sassi_ctx_create(0, s, 1)
    assert e.value.status == sassi.SASSI_EINVAL
    s["pc"] = [0x10, 0x20]
    s[0]["flags"] = 1 | 4                        # branch that also accesses memory
    with pytest.raises(sassi.SassiError) as e:
        sassi.sassi_ctx_create(0, s, 1)
    assert e.value.status == sassi.SASSI_EINVAL

"""CPU-side checks of the C ABI: the library builds for sm_100a, loads without a
GPU, exports every symbol include/agnn.h declares, and its pure host logic
(agnn_partition, argument validation) is bit-exact with the oracle."""
from __future__ import annotations

import ctypes
import re
import os

import numpy as np
import pytest

import oracle
from paper_conf_sc_bestarglzcgssci23_b200 import agnn, _build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "agnn.h")).read()
    return sorted(set(re.findall(r"^(?:agnn_status|void|uint64_t|size_t|const char\*)\s+(agnn_\w+)\(",
                                 src, flags=re.M)))


def test_header_and_binding_agree():
    assert declared_symbols() == sorted(agnn.EXPORTS)


def test_plan_options_layout_matches_header():
    """agnn_plan_options (include/agnn.h) and the ctypes binding: same fields, order, types."""
    src = open(os.path.join(ROOT, "include", "agnn.h")).read()
    end = src.index("} agnn_plan_options;")
    body = src[src.rindex("typedef struct {", 0, end):end]
    body = re.sub(r"/\*.*?\*/", "", body, flags=re.S)
    fields = re.findall(r"int32_t\s+(\w+);", body)
    assert fields == [f for f, _ in agnn.PlanOptions._fields_]
    assert all(t is ctypes.c_int32 for _, t in agnn.PlanOptions._fields_)


def test_library_exports_every_declared_symbol():
    L = agnn.lib()
    for name in declared_symbols():
        assert hasattr(L, name), name


def test_library_is_sm100a_only():
    out = os.popen(f"cuobjdump --list-elf {_build.AGNN_SO} 2>&1").read()
    arches = set(re.findall(r"sm_(\d+a?)", out))
    assert arches == {"100a"}, out


def test_status_strings():
    L = agnn.lib()
    assert L.agnn_status_string(0) == b"AGNN_OK"
    assert L.agnn_status_string(5) == b"AGNN_EUNSUPPORTED"


@pytest.mark.parametrize("world", [1, 2, 3, 4, 8])
@pytest.mark.parametrize("c_v", [0, 4, 17])
def test_partition_bit_exact_with_oracle(world, c_v):
    rng = np.random.default_rng(world * 31 + c_v)
    for n in (1, 5, 1000, 4096):
        deg = rng.zipf(1.8, n).clip(max=5000) if n > 5 else rng.integers(0, 4, n)
        rp = np.concatenate([[0], np.cumsum(deg)]).astype(np.int64)
        np.testing.assert_array_equal(agnn.partition(rp, world, c_v), oracle.partition(rp, world, c_v))


def test_partition_rejects_bad_arguments():
    with pytest.raises(agnn.AgnnError):
        agnn.partition(np.array([0, 1], np.int64), 0)


def test_model_create_rejects_bad_descriptors():
    L = agnn.lib()
    h = ctypes.c_void_p()
    # NULL plan -> EINVAL without touching the device
    d = agnn.layer_desc("gat", 64, 64, 3)
    assert L.agnn_model_create(None, 1, ctypes.byref(d), ctypes.byref(h)) == 1

"""Host-side checks of bench.py's algorithmic byte model.

The roofline the bench reports divides these bytes by the measured pass time, so
the per-edge / per-row figures must be the ones the design states: GAT at C5
(k' = 128, 4 heads, fp32) moves 532 B per stored entry in the forward, 580 B in
the factored backward and 1108 B in the unfactored one.
"""
from __future__ import annotations

import dataclasses
import importlib.util
import os

import pytest

from paper_conf_sc_bestarglzcgssci23_b200 import gen

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench():
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    mod = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(mod)
    return mod


def test_gat_c5_bytes_per_edge():
    b = _bench()
    w = gen.CONFIGS["C5"]
    pb = b.pass_bytes(w, 1000, 10)
    assert pb["fwd"][1] == 4 + 128 * 4 + 4 * 4 == 532
    assert pb["bwd"][1] == 4 + 128 * 4 + 16 * 4 == 580          # factored: G_i + rec_i
    assert pb["bwd"][0] == 580 * 1000 + pb["bwd"][2] * 10
    assert b.pass_bytes(w, 1000, 10, factored_mode=0)["bwd"][1] == 4 + 2 * 128 * 4 + 20 * 4 == 1108


def test_gat_bf16_storage_bytes():
    b = _bench()
    w = dataclasses.replace(gen.CONFIGS["C5"], prec="bf16")
    pb = b.pass_bytes(w, 1, 0)
    assert pb["fwd"][1] == 4 + 128 * 2 + 16 == 276
    assert pb["bwd"][1] == 4 + 128 * 2 + 64 == 324


@pytest.mark.parametrize("cfg,per_edge", [("C3", 4 + 2 * 128 * 4 + 16), ("C4", 4 + 2 * 256 * 4)])
def test_agnn_va_bytes(cfg, per_edge):
    b = _bench()
    w = gen.CONFIGS[cfg]
    assert b.pass_bytes(w, 1, 0)["bwd"][1] == per_edge


def test_factored_mode_selection():
    b = _bench()
    c5, c2 = gen.CONFIGS["C5"], gen.CONFIGS["C2"]   # k' = 128 / k' = 64
    assert b.gat_factored(c5) and not b.gat_factored(c2)
    assert b.gat_factored(c5, 2) and b.gat_factored(c2, 2)
    assert not b.gat_factored(c5, 0)

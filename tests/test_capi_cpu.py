"""C-ABI library checks that need no GPU: libinsta.so loads, exports every symbol
include/insta.h declares, and its host levelizer matches the oracle's
independent levelizer bit for bit."""
import os
import re

import numpy as np
import pytest

import oracle
import paper_conf_dac_lugklr25_b200 as insta
from paper_conf_dac_lugklr25_b200 import _capi, synth
from tests import bruteforce as bf

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_symbols():
    src = open(os.path.join(ROOT, "include", "insta.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(insta_[a-z_]+)\s*\(", src)))


def test_library_exports_every_declared_symbol():
    lib = _capi.load()
    declared = _declared_symbols()
    assert len(declared) >= 12
    for name in declared:
        assert hasattr(lib, name), name
        assert name in _capi.SIGNATURES, name
    assert "sm_100a" in insta.version()


def test_library_is_built_for_sm100a():
    import subprocess
    out = subprocess.run(["cuobjdump", "--list-elf", _capi.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def _same(a, b):
    for k in ("level", "order", "fanin_ptr", "fanin_arc", "fanout_ptr", "fanout_arc"):
        assert np.array_equal(a[k], b[k]), k
    assert a["num_levels"] == b["num_levels"]


@pytest.mark.parametrize("seed", range(10))
def test_levelize_bit_exact_vs_oracle_tiny(seed):
    g = bf.tiny_dag(seed, n_pins=9)
    _same(insta.levelize(g.num_pins, g.arc_from, g.arc_to), oracle.levelize(g.num_pins, g.arc_from, g.arc_to))


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3"])
def test_levelize_bit_exact_vs_oracle_configs(cfg):
    g = synth.generate(cfg)
    _same(insta.levelize(g.num_pins, g.arc_from, g.arc_to), oracle.levelize(g.num_pins, g.arc_from, g.arc_to))


def test_levelize_edge_cases():
    # no arcs: every pin is a level-0 source
    r = insta.levelize(5, np.zeros(0, np.int32), np.zeros(0, np.int32))
    assert r["num_levels"] == 1 and list(r["order"]) == [0, 1, 2, 3, 4]
    # empty graph
    r = insta.levelize(0, np.zeros(0, np.int32), np.zeros(0, np.int32))
    assert r["num_levels"] == 0
    # parallel arcs and a long chain
    r = insta.levelize(4, [0, 0, 1, 2], [1, 1, 2, 3])
    assert list(r["level"]) == [0, 1, 2, 3] and list(r["fanin_arc"]) == [0, 1, 2, 3]


def test_levelize_errors():
    with pytest.raises(insta.InstaError, match="E_CYCLE"):
        insta.levelize(3, [0, 1, 2], [1, 2, 0])
    with pytest.raises(insta.InstaError, match="E_CYCLE"):
        insta.levelize(2, [1], [1])
    with pytest.raises(insta.InstaError, match="E_ARG"):
        insta.levelize(2, [0], [5])


def test_graph_create_rejects_bad_descriptors_before_touching_a_device():
    import types
    g = bf.tiny_dag(2)
    bad = types.SimpleNamespace(**vars(g))
    bad.arc_sigma = np.array(g.arc_sigma, np.float32)
    bad.arc_sigma[0, 0] = -1.0
    with pytest.raises(insta.InstaError, match="E_ARG"):
        insta.Graph(bad)
    dup = types.SimpleNamespace(**vars(g))
    dup.ep_pin = np.array([0, 0], np.int32)
    dup.ep_rat = np.zeros((2, 2), np.float32)
    with pytest.raises(insta.InstaError, match="duplicate"):
        insta.Graph(dup)

"""CPU tests of the generic space IR front half: the
library validates an IR description, assigns levels (the level-set rule,
PAPER.md:1576-1594) and compiles the generated CUDA for sm_100a with NVRTC
-- all without a GPU.  Levels must agree with the oracle's own assignment
(oracle/ir.py); malformed descriptions must be rejected with a message."""
from __future__ import annotations

import os
import sys

import pytest

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import beast_inputs as bi  # noqa: E402
import ir_specs  # noqa: E402
import oracle  # noqa: E402
from oracle import ir as oir  # noqa: E402


@pytest.fixture(scope="module")
def beast():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_luszczekgkdd16_b200 as b
    return b


def _specs():
    out = dict(ir_specs.toy_specs())
    out["gemm_tiny_S_10"] = ir_specs.gemm_spec(oracle.resolve(bi.tiny("S", 1, 0)), "S")
    return out


@pytest.mark.parametrize("name", sorted(_specs()))
def test_ir_compiles_and_levels_agree(beast, name):
    spec = _specs()[name]
    with beast.IRSpace(spec) as sp:
        want = {k: v for k, v in oir.levels(spec).items() if k not in spec["constants"]}
        assert sp.levels() == want
        src = sp.source
        assert "ir_count" in src and "ir_emit" in src
        for c, _ in spec["constraints"]:
            assert c in src


@pytest.mark.parametrize("bad", [
    {"iterators": [["a", "0", "b", "1"], ["b", "0", "3", "1"]]},                 # later iterator in a range
    {"iterators": [["a", "0", "3", "1"]], "derived": [["x", "y + 1"], ["y", "a"]]},   # used before declared
    {"iterators": [["a", "0", "3", "1"]], "constraints": [["c", "a +* 2"]]},          # does not compile
    {"iterators": [["ir_x", "0", "3", "1"]]},                                          # reserved name
    {"iterators": [["a", "0", "3", "1"], ["a", "0", "3", "1"]]},                       # duplicate
    {"iterators": [["a", "0", "3", "1"]], "constraints": [["c", "zz > 1"]]},           # unknown name
])
def test_ir_rejects_malformed(beast, bad):
    spec = dict(constants={}, derived=[], constraints=[])
    spec.update(bad)
    with pytest.raises(beast.BeastError):
        beast.IRSpace(spec)

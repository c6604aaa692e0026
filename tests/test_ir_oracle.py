"""Pins of the generic-IR oracle (oracle/ir.py) -- CPU.

* The paper's GEMM space written in the IR (tests/ir_specs.gemm_spec) must
  enumerate exactly like the hand-written canonical nest oracle.nest on every
  tiny configuration, the micro space and fuzz spaces: survivor list (packed
  into the record layout of include/beast.h), per-level visits and
  first-failing rejections (the level-set rule).
* Toy specs must give the survivor list of a by-definition Python brute
  force (dependent-range product, all constraints at the leaf).
* Level assignment on hand-checked cases.
"""
from __future__ import annotations

import os
import sys

import numpy as np
import pytest

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import beast_inputs as bi  # noqa: E402
import ir_specs  # noqa: E402
import oracle  # noqa: E402
from oracle import ir as oir  # noqa: E402


def pack(rec: np.ndarray) -> np.ndarray:
    """IR tuples (15 int64 per survivor, Fig 11 order) -> (hi, lo) words."""
    r = rec.astype(np.uint64)
    hi = (r[:, 0] << 52) | (r[:, 1] << 40) | (r[:, 2] << 28) | (r[:, 3] << 16) | (r[:, 4] << 4) | \
         (r[:, 5] << 1) | r[:, 6]
    lo = (r[:, 7] << 52) | (r[:, 8] << 40) | (r[:, 9] << 28) | (r[:, 10] << 16) | (r[:, 11] << 3) | \
         (r[:, 12] << 2) | (r[:, 13] << 1) | r[:, 14]
    return np.stack([hi, lo], 1)


def _gemm_check(desc):
    res = oracle.resolve(desc)
    got = oir.run(ir_specs.gemm_spec(res, desc["precision"]), records=True)
    ref = oracle.nest(desc, records=True)
    assert got["survivors"] == ref["survivors"]
    assert got["visits"] == ref["visits"]
    assert got["rejected"] == ref["rejected"]
    assert np.array_equal(pack(got["records"]), ref["records"].astype(np.uint64))


@pytest.mark.parametrize("p", bi.PRECISIONS)
@pytest.mark.parametrize("ta,tb", bi.TRANSPOSES)
def test_gemm_ir_equals_nest_tiny(p, ta, tb):
    _gemm_check(bi.tiny(p, ta, tb))


@pytest.mark.parametrize("seed", range(8))
def test_gemm_ir_equals_nest_fuzz(seed):
    _gemm_check(bi.fuzz_space(seed, max_bound=12))


def test_gemm_ir_equals_nest_micro():
    _gemm_check(bi.micro("C"))


@pytest.mark.parametrize("name", sorted(ir_specs.toy_specs()))
def test_toy_equals_brute(name):
    spec = ir_specs.toy_specs()[name]
    got = oir.run(spec, records=True)
    want = ir_specs.brute(spec)
    assert [tuple(x) for x in got["records"].tolist()] == want
    assert got["survivors"] == len(want)
    # every visit either continues or is rejected by exactly one constraint
    lev = oir.levels(spec)
    its = [i[0] for i in spec["iterators"]]
    for d in range(len(its)):
        rej_here = sum(r for (c, _), r in zip(spec["constraints"], got["rejected"]) if lev[c] == d)
        passed = got["visits"][d] - rej_here
        nxt = got["visits"][d + 1] if d + 1 < len(its) else got["survivors"]
        if d + 1 == len(its):
            assert passed == nxt


def test_levels_hand_checked():
    spec = ir_specs.toy_specs()["multiples"]
    lev = oir.levels(spec)
    assert lev["a"] == 0 and lev["b"] == 1 and lev["c"] == 2
    assert lev["p"] == 1 and lev["q"] == 2
    assert lev["odd_a"] == 0 and lev["big"] == 1 and lev["c_div"] == 2 and lev["q_mod"] == 2
    lev = oir.levels(ir_specs.toy_specs()["empty_inner"])
    assert lev["const_ok"] == -1 and lev["first"] == 0 and lev["t_neg"] == 2
    g = oir.levels(ir_specs.gemm_spec(oracle.resolve(bi.tiny("D")), "D"))
    # the canonical hoisting of SURVEY §8(c): L2, L4, L5, L6, L9, L11 (0-based 1, 3, 4, 5, 8, 10)
    assert g["over_max_threads"] == 1 and g["partial_warps"] == 1
    assert g["over_max_regs_per_thread"] == 3 and g["low_occupancy_regs"] == 3
    assert g["over_max_shmem"] == 4 and g["low_occupancy_shmem"] == 4
    assert g["low_fmas"] == 5
    assert g["cant_reshape_a1"] == 8 and g["cant_reshape_a2"] == 8
    assert g["cant_reshape_b1"] == 10 and g["cant_reshape_b2"] == 10

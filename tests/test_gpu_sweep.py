"""GPU parity of the batched sweep (beast_sweep_count).

A sweep counts many independent spaces in one call, their passes running
concurrently on internal streams.  The bar is the same as for beast_count:
bit-exact survivor counts, per-level visits and first-failing rejections,
here against the oracle-written goldens (tests/golden/expected.json, by
scripts/make_golden.py from oracle/ alone) for the 32 configurations the
paper tunes one at a time (4 precisions x 4 transposes x {K40c, B200};
P:898-900, Fig 10), and against the oracle nest run here for
small spaces.
"""
from __future__ import annotations

import json
import os

import pytest

import beast_inputs as bi
import oracle

pytestmark = pytest.mark.gpu

GOLDEN = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "expected.json")))
SWEEP_KEYS = ["%s_%s_%d%d" % (dev, p, ta, tb) for dev in ("k40c", "b200") for p in bi.PRECISIONS
              for ta, tb in bi.TRANSPOSES]


@pytest.fixture(scope="module")
def beast():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_luszczekgkdd16_b200 as b
    return b


def test_sweep_32_configs_against_goldens(beast):
    assert all(k in GOLDEN for k in SWEEP_KEYS)
    spaces = [beast.Space.from_desc(GOLDEN[k]["space"]) for k in SWEEP_KEYS]
    try:
        counts, stats = beast.sweep(spaces, stats=True)
        for k, n, st in zip(SWEEP_KEYS, counts, stats):
            g = GOLDEN[k]
            assert n == g["survivors"] == st["survivors"], k
            assert st["visits"] == g["visits"], k
            assert st["rejected"] == g["rejected"], k
            assert st["prefixes"] == g["prefixes"] and st["valid_a"] == g["valid_a"], k
        # replayed (captured) passes, counts only, twice: same answers
        for _ in range(2):
            assert beast.sweep(spaces) == [GOLDEN[k]["survivors"] for k in SWEEP_KEYS]
    finally:
        for sp in spaces:
            sp.close()


def test_sweep_small_spaces_against_oracle(beast):
    descs = [bi.tiny(p, ta, tb) for p in bi.PRECISIONS for ta, tb in bi.TRANSPOSES]
    descs += [bi.fuzz_space(s) for s in range(24)] + [bi.micro("C")]
    spaces = [beast.Space.from_desc(d) for d in descs]
    try:
        counts, stats = beast.sweep(spaces, stats=True)
        for d, n, st in zip(descs, counts, stats):
            ref = oracle.nest(d, digest=False)
            assert n == ref["survivors"]
            assert st["visits"] == ref["visits"] and st["rejected"] == ref["rejected"]
        assert beast.sweep(spaces) == counts
    finally:
        for sp in spaces:
            sp.close()


def test_sweep_matches_single_counts_and_mixes_with_them(beast):
    descs = [bi.tiny("D"), bi.named("headline"), bi.fuzz_space(7)]
    spaces = [beast.Space.from_desc(d) for d in descs]
    try:
        single = [sp.count() for sp in spaces]
        assert beast.sweep(spaces) == single
        assert [sp.count() for sp in spaces] == single     # handles stay usable after a sweep
        assert beast.sweep(spaces[::-1]) == single[::-1]
    finally:
        for sp in spaces:
            sp.close()


def test_sweep_edge_cases(beast):
    assert beast.sweep([]) == []
    sp = beast.Space.from_desc(bi.tiny("D"))
    try:
        with pytest.raises(beast.BeastError):
            beast.sweep([sp, sp])                             # a handle's passes are serial
        empty = bi.make_space(dict(bi.K40C_DEVICE, max_threads_per_block=16), "D", bounds=8)
        with beast.Space.from_desc(empty) as e:
            assert beast.sweep([sp, e]) == [1824, 0]
    finally:
        sp.close()

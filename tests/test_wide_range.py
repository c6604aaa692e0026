"""The library's whole admitted input range (include/beast.h,
beast_space_create: threads_per_block up to 65535, float_size up to 1024,
max_blocks_per_multi_processor up to 65534, min_threads up to 2^30,
min_fmas up to 2^20, limits up to 2^31 - 1, bounds up to 4095) on the
oracle side (CPU): the wide-fuzz fixture (scripts/make_wide_fuzz.py, oracle
only) is reproducible, covers that range, and equals the oracle's current
output; the oracle's independent pins (brute force, analytic counter) hold
there too.  The GPU side of the same spaces is tests/test_gpu_parity.py
(test_fuzz_wide, the ext_* goldens)."""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import beast_inputs as bi
import oracle
import oracle.analytic

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
with open(os.path.join(ROOT, "tests", "golden", "wide_fuzz.json")) as _f:
    WIDE = json.load(_f)["spaces"]
A = bi.ADMITTED


def test_wide_fixture_is_the_generator():
    assert sorted(int(k) for k in WIDE) == list(range(200, 400))
    for k, e in WIDE.items():
        assert e["attempt"] is not None, k
        assert bi.fuzz_space_wide(int(k), e["attempt"]) == e["space"], k


def test_wide_fixture_covers_admitted_range(golden_expected):
    sp = [e["space"] for e in WIDE.values()]

    def has(field, value):
        return any(s[field] == value for s in sp)

    assert has("max_threads_per_block", A["max_threads_per_block"])
    assert has("float_size", A["float_size"])
    assert has("max_blocks_per_multi_processor", A["max_blocks_per_multi_processor"])
    assert has("min_threads_per_multi_processor", A["min_threads_per_multi_processor"])
    assert has("min_fmas_per_load", A["min_fmas_per_load"])
    for f in ("max_shared_mem_per_block", "max_shmem_per_multi_processor", "max_regs_per_block",
              "max_registers_per_multi_processor", "max_registers_per_thread"):
        assert has(f, A["int32"]), f
    assert any(s[b] == A["bound"] for s in sp for b in bi.BOUND_FIELDS)
    assert has("warp_size", 1) and has("warp_size", 64)
    with_surv = [e for e in WIDE.values() if e["survivors"]]
    assert len(with_surv) >= 20
    assert sum(e["t_max"] > 1024 for e in with_surv) >= 3
    # survivors above 1024 threads per block in the fixture's spaces with the
    # widest float / limit values
    assert any(e["survivors"] and e["space"]["max_threads_per_block"] == A["max_threads_per_block"]
               for e in WIDE.values())
    # the extreme goldens: threads_per_block >= 16384 among the survivors
    for key in ("ext_bigT_D_00", "ext_bigT_S_11"):
        e = golden_expected[key]
        assert e["survivors"] > 0
        hi = int(e["first"][0], 16)
        assert (hi >> 52) * ((hi >> 40) & 0xFFF) >= 4096, key
    hi = int(golden_expected["ext_bigT_D_00"]["first"][0], 16)
    assert (hi >> 52) * ((hi >> 40) & 0xFFF) >= 16384


@pytest.mark.parametrize("seed", [s for s in range(200, 400, 9)])
def test_wide_fixture_matches_oracle(seed):
    e = WIDE[str(seed)]
    r = oracle.nest(e["space"], threads=os.cpu_count(), digest=True)
    assert r["survivors"] == e["survivors"] and r["visits"] == e["visits"]
    assert r["rejected"] == e["rejected"] and "0x%016x" % r["digest"] == e["digest"]


@pytest.mark.parametrize("seed", [s for s in range(200, 400, 11)])
def test_analytic_equals_nest_wide(seed):
    """Pin P5 over the admitted range: the divisor-based counter (no inner
    loops) equals the canonical nest."""
    e = WIDE[str(seed)]
    if e["n_canon"] > 100_000_000:
        pytest.skip("large")
    a = oracle.analytic.count(e["space"])
    assert a["visits"] == e["visits"] and a["rejected"] == e["rejected"]


@pytest.mark.parametrize("seed", range(200, 240))
def test_brute_force_wide_limits(seed):
    """Pin P1 over the admitted range of the device limits and thresholds
    (bounds clamped to <= 6 so that the full product is brute-forceable)."""
    e = WIDE[str(seed)]
    sp = dict(e["space"])
    for b in bi.BOUND_FIELDS:
        sp[b] = min(sp[b], 6)
    br = oracle.brute(sp)
    ne = oracle.nest(sp, records=True)
    assert br["survivors"] == ne["survivors"]
    assert np.array_equal(np.asarray(br["records"], np.uint64).reshape(-1, 2), ne["records"])


def _shape_sums(shapes):
    return (sum(m * c for (m, n), c in shapes.items()), sum(m * n * c for (m, n), c in shapes.items()))


@pytest.mark.parametrize("desc", [bi.tiny(p, a, b) for p in bi.PRECISIONS for a, b in bi.TRANSPOSES] +
                         [bi.fuzz_space(s) for s in range(10)] +
                         [WIDE[str(s)]["space"] for s in (203, 205, 213, 226, 233)])
def test_grid_shape_histograms_pin_to_nest(desc):
    """The analytic counter's A / B grid-shape histograms (the reference for
    beast_stats.formed) reproduce the nest's L8-L11 visits: sum RA_m = V8,
    sum RA_m * RA_n = V9, sum RB_m = V10, sum RB_m * RB_n = V11."""
    sh = oracle.analytic.count(desc, shapes=True)
    v = oracle.nest(desc)["visits"]
    assert _shape_sums(sh["a_shapes"]) == (v[7], v[8])
    assert _shape_sums(sh["b_shapes"]) == (v[9], v[10])

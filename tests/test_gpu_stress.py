"""GPU stress: many replays of the captured pass must give the golden list
every time.  The tiled evaluation synchronises its warps through shared
memory (tile build, chunk map, candidate rings) and claims tiles and appends
results with global atomics whose order changes from run to run, so a
missing barrier or a lost update would show up as an occasional wrong count
or list.  (compute-sanitizer is closed on this GPU pool; this is the
run-time check that replaces its racecheck / synccheck.)  Digests and counts
come from tests/golden/expected.json (written by the oracle alone)."""
from __future__ import annotations

import pytest

import beast_inputs as bi

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def beast():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_luszczekgkdd16_b200 as b
    return b


CASES = [("k40c_D_00", lambda: bi.k40c("D", 0, 0), 200), ("k40c_Z_11", lambda: bi.k40c("Z", 1, 1), 200),
         ("b200_D_10", lambda: bi.b200("D", 1, 0), 50), ("b200_C_01", lambda: bi.b200("C", 0, 1), 30)]


@pytest.mark.parametrize("key,make,reps", CASES, ids=[c[0] for c in CASES])
def test_replays_match_golden(beast, golden_expected, key, make, reps):
    import torch
    e = golden_expected[key]
    with beast.Space.from_desc(make()) as sp:
        n = sp.count()
        assert n == e["survivors"]
        out = torch.empty((max(n, 1), 2), dtype=torch.uint64, device="cuda")
        bad = []
        for r in range(reps):
            w = beast.beast_enumerate(sp.handle, out)
            d = "0x%016x" % beast.beast_digest(out[:w]) if w else "0x%016x" % 0
            if w != e["survivors"] or (w and d != e["digest"]):
                bad.append((r, w, d))
            c = sp.count()
            if c != e["survivors"]:
                bad.append((r, "count", c))
        assert not bad, bad[:5]

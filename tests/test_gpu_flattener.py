"""GPU parity of the round-1 global-flattener path (`BEAST_FLATTENER=1`:
k_bucket_count + k_bucket_place + k_eval per stage), kept as the A/B
reference of the tiled evaluation (`k_tile_eval`, the default; DESIGN.md
§6): on the same spaces both paths must give the same list, counts, visits,
rejections and evaluation evidence, and the small ones the oracle's.  The
library reads the switch when a handle first runs, so each path gets handles
of its own."""
from __future__ import annotations

import os

import numpy as np
import pytest

import json

import beast_inputs as bi
import oracle

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
with open(os.path.join(ROOT, "tests", "golden", "wide_fuzz.json")) as _f:
    WIDE = json.load(_f)["spaces"]

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


def _run(beast, desc, flattener):
    old = os.environ.get("BEAST_FLATTENER")
    os.environ["BEAST_FLATTENER"] = "1" if flattener else "0"
    try:
        with beast.Space.from_desc(desc) as sp:
            rec, st = sp.enumerate(stats=True)
            got = rec.cpu().numpy().copy()
            n = sp.count()
    finally:
        if old is None:
            os.environ.pop("BEAST_FLATTENER", None)
        else:
            os.environ["BEAST_FLATTENER"] = old
    return got, st, n


SPACES = ["tiny", "micro", "headline"] + [("fuzz", s) for s in (3, 17, 42, 101)] + [("wide", s) for s in (200, 257)]


def _desc(which):
    if isinstance(which, tuple):
        kind, seed = which
        return bi.fuzz_space(seed) if kind == "fuzz" else bi.fuzz_space_wide(seed, WIDE[str(seed)]["attempt"])
    return bi.named(which)


@pytest.mark.parametrize("which", SPACES, ids=lambda w: w if isinstance(w, str) else "%s%d" % w)
def test_flattener_path_equals_tiled(beast, which):
    desc = _desc(which)
    g1, s1, n1 = _run(beast, desc, flattener=True)
    g0, s0, n0 = _run(beast, desc, flattener=False)
    assert n1 == n0 == len(g0) == len(g1)
    assert np.array_equal(g0, g1)
    for k in ("visits", "rejected", "formed", "survivors", "valid_a", "tuples"):
        assert s0[k] == s1[k], k
    # rows checked exactly may differ: in a tile a lane whose job has shorter
    # rows than its chunk's first also scans the extra blocks, and a zero half
    # found there is queued and rejected by the exact check (t <= L)
    a1_pass = (s0["visits"][8] - s0["rejected"][8], s0["visits"][10] - s0["rejected"][9])
    for st in (s0, s1):
        assert st["checked"][0] >= a1_pass[0] and st["checked"][1] >= a1_pass[1]
    if s0["points"] < 3e8:
        ref = oracle.nest(desc, threads=os.cpu_count(), records=True)
        want = np.stack([ref["records"][:, 1], ref["records"][:, 0]], 1) if ref["survivors"] else np.zeros((0, 2), np.uint64)
        assert np.array_equal(g0, want)
        assert s0["visits"] == ref["visits"] and s0["rejected"] == ref["rejected"]

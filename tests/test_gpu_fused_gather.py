"""GPU parity of the fused survivor gather:
beast_enumerate_stage + beast_write_at.

Each (virtual) rank stages its shard, the per-rank record counts form the
device array every rank's write-out reads its base offset from, and every
shard's records are stored into ONE buffer at that offset.  On one GPU the
ranks are virtual (one handle each, all writing into a local buffer); the
bar is the multi-GPU one: the buffer equals the world-1 canonical list
bit-exactly (memcmp against the oracle for small spaces, digest and count
against tests/golden for full-size ones).  The same two calls run over
NVLink with rank 0's symmetric-memory buffer in dist.FusedGather.
"""
from __future__ import annotations

import json
import os

import numpy as np
import pytest

import beast_inputs as bi
import oracle

pytestmark = pytest.mark.gpu

GOLDEN = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "expected.json")))


@pytest.fixture(scope="module")
def beast():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_luszczekgkdd16_b200 as b
    return b


def _fused_virtual(beast, desc, world, capacity=None):
    import torch
    spaces = [beast.Space.from_desc(desc) for _ in range(world)]
    try:
        d_counts = torch.zeros(world, dtype=torch.int64, device="cuda")
        counts = []
        for r, sp in enumerate(spaces):
            counts.append(beast.beast_enumerate_stage(sp.handle, d_counts[r:r + 1], r, world))
        total = sum(counts)
        assert int(d_counts.sum().item()) == total
        cap = max(total, 1) if capacity is None else capacity
        out = torch.full((cap, 2), -1, dtype=torch.int64, device="cuda")
        bases = [beast.beast_write_at(sp.handle, out.data_ptr(), cap, d_counts, r, world)
                 for r, sp in enumerate(spaces)]
        torch.cuda.synchronize()
        assert bases == list(np.cumsum([0] + counts[:-1]))
        return out[:total].view(torch.uint64), counts
    finally:
        for sp in spaces:
            sp.close()


@pytest.mark.parametrize("world", [1, 2, 3, 8])
@pytest.mark.parametrize("name", ["tiny_D", "tiny_C", "micro"])
def test_fused_virtual_ranks_small(beast, name, world):
    desc = bi.micro("C") if name == "micro" else bi.tiny(name[-1])
    got, counts = _fused_virtual(beast, desc, world)
    ref = oracle.nest(desc, records=True)
    want = np.stack([ref["records"][:, 1], ref["records"][:, 0]], 1) if ref["survivors"] else np.zeros((0, 2), np.uint64)
    assert np.array_equal(got.cpu().numpy(), want)


@pytest.mark.parametrize("world", [2, 8])
@pytest.mark.parametrize("key", ["k40c_D_00", "b200_C_11", "widened256_k40c_D_00"])
def test_fused_virtual_ranks_full(beast, key, world):
    g = GOLDEN[key]
    got, counts = _fused_virtual(beast, g["space"], world)
    assert got.shape[0] == g["survivors"]
    assert "0x%016x" % beast.beast_digest(got) == g["digest"]


def test_fused_gather_single_process(beast):
    from paper_conf_ipps_luszczekgkdd16_b200 import dist as bdist
    desc = bi.named("headline")
    with beast.Space.from_desc(desc) as sp:
        n = sp.count()
        fg = bdist.FusedGather(n)
        for _ in range(2):
            assert fg.run(sp) == n
        rec = sp.enumerate()
        assert np.array_equal(fg.buf[:n].view(__import__("torch").uint64).cpu().numpy(), rec.cpu().numpy())


def test_fused_errors(beast):
    import torch
    desc = bi.tiny("D")
    with beast.Space.from_desc(desc) as sp:
        d = torch.zeros(2, dtype=torch.int64, device="cuda")
        out = torch.empty((4000, 2), dtype=torch.int64, device="cuda")
        with pytest.raises(beast.BeastError):                        # nothing staged yet
            beast.beast_write_at(sp.handle, out.data_ptr(), 4000, d, 0, 1)
        n = beast.beast_enumerate_stage(sp.handle, d[:1], 0, 1)
        assert n == 1824
        with pytest.raises(beast.BeastError):                        # capacity too small
            beast.beast_write_at(sp.handle, out.data_ptr(), n - 1, d, 0, 1)
        d[0] = n + 16
        with pytest.raises(beast.BeastError):                        # count mismatch
            beast.beast_write_at(sp.handle, out.data_ptr(), 4000, d, 0, 1)
        d[0] = n
        sp.count()                                                   # another pass: stage is gone
        with pytest.raises(beast.BeastError):
            beast.beast_write_at(sp.handle, out.data_ptr(), 4000, d, 0, 1)

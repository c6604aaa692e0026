"""GPU parity: the CUDA path (through the C ABI) against the oracle.

Bar: integer work, so bit-exact — survivor count,
canonically ordered packed list (memcmp or the order-sensitive digest),
per-level visits and first-failing rejection counts.  Small spaces run the
oracle here; full-size spaces compare with tests/golden/expected.json, which
scripts/make_golden.py wrote from the oracle alone.
"""
from __future__ import annotations

import os
import random

import json

import numpy as np
import pytest

import beast_inputs as bi
import oracle
import oracle.analytic

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


def _oracle_lohi(rec):
    return np.stack([rec[:, 1], rec[:, 0]], axis=1) if len(rec) else np.zeros((0, 2), np.uint64)


def _run(beast, desc, rank=0, world=1, stats=True):
    with beast.Space.from_desc(desc) as sp:
        rec, st = sp.enumerate(rank=rank, world=world, stats=True)
        got = rec.cpu().numpy().copy()
        dig = beast.beast_digest(rec) if len(rec) else 0
        n = sp.count(rank=rank, world=world)
    return got, st, dig, n


def _formed(shapes):
    """Points the packed scan forms over grids of the given shape histogram
    (include/beast.h, beast_stats.formed): a grid of m x n points is
    min(m, n) rows of max(m, n) points, each row run in whole 16-point
    blocks."""
    tot = 0
    for (m, n), c in shapes.items():
        tot += c * min(m, n) * 16 * ((max(m, n) + 15) // 16)
    return tot


def _check_evaluated(desc, st, exact=True):
    """The instrumented run formed every canonical A and B grid point (and
    only the row padding on top): formed == the oracle's grid shapes in the
    row layout (exact) or visits <= formed <= visits + 15 rows (bound)."""
    v, rej = st["visits"], st["rejected"]
    if exact:
        sh = oracle.analytic.count(desc, shapes=True)
        assert st["formed"] == [_formed(sh["a_shapes"]), _formed(sh["b_shapes"])]
    assert v[8] <= st["formed"][0] <= v[8] + 15 * v[7]
    assert v[10] <= st["formed"][1] <= v[10] + 15 * v[9]
    # every row with a point passing a1 (b1) was checked exactly
    assert st["checked"][0] >= v[8] - rej[8] and st["checked"][1] >= v[10] - rej[9]


def _check_small(beast, desc):
    got, st, dig, n = _run(beast, desc)
    ref = oracle.nest(desc, records=True)
    want = _oracle_lohi(ref["records"])
    assert got.shape == want.shape, (got.shape, want.shape)
    assert np.array_equal(got, want)
    assert n == ref["survivors"] == st["survivors"]
    assert st["visits"] == ref["visits"], (st["visits"], ref["visits"])
    assert st["rejected"] == ref["rejected"], (st["rejected"], ref["rejected"])
    if len(got):
        assert dig == ref["digest"]
    _check_evaluated(desc, st)


@pytest.mark.parametrize("p", bi.PRECISIONS)
@pytest.mark.parametrize("ta,tb", bi.TRANSPOSES)
def test_tiny(beast, p, ta, tb):
    _check_small(beast, bi.tiny(p, ta, tb))


def test_micro(beast):
    _check_small(beast, bi.micro("C"))


@pytest.mark.parametrize("seed", range(200))
def test_fuzz(beast, seed):
    _check_small(beast, bi.fuzz_space(seed))


@pytest.mark.parametrize("seed", range(200, 400))
def test_fuzz_wide(beast, seed):
    """The library's whole admitted input range (beast_inputs.fuzz_space_wide:
    threads_per_block up to 65535, float_size up to 1024, max_blocks up to
    65534, thresholds up to 2^30 / 2^20, limits up to 2^31 - 1, bounds up to
    4095), bit-exact against the oracle run here (and its fixture)."""
    e = WIDE[str(seed)]
    desc = bi.fuzz_space_wide(seed, e["attempt"])
    assert desc == e["space"]
    got, st, dig, n = _run(beast, desc)
    assert n == st["survivors"] == e["survivors"]
    assert st["visits"] == e["visits"] and st["rejected"] == e["rejected"]
    if n:
        assert "0x%016x" % dig == e["digest"]
    ref = oracle.nest(desc, threads=os.cpu_count(), records=True)
    assert np.array_equal(got, _oracle_lohi(ref["records"]))
    _check_evaluated(desc, st, exact=e["n_canon"] < 50_000_000)


def test_empty_space(beast):
    # warp_size larger than any threads_per_block: L2 rejects everything
    desc = bi.make_space(dict(bi.K40C_DEVICE, max_threads_per_block=16), "D", bounds=8)
    got, st, dig, n = _run(beast, desc)
    assert n == 0 and got.shape == (0, 2) and st["survivors"] == 0
    _check_small(beast, desc)


def test_degenerate_bounds_one(beast):
    _check_small(beast, bi.make_space(bi.K40C_DEVICE, "S", bounds=1))
    _check_small(beast, bi.make_space(dict(bi.K40C_DEVICE, warp_size=1), "S", bounds=1))


def test_headline_bit_exact(beast):
    desc = bi.headline()
    got, st, dig, n = _run(beast, desc)
    ref = oracle.nest(desc, threads=os.cpu_count(), records=True)
    assert np.array_equal(got, _oracle_lohi(ref["records"]))
    assert st["visits"] == ref["visits"] and st["rejected"] == ref["rejected"]
    assert dig == ref["digest"] and n == 1_207_600
    _check_evaluated(desc, st)


GOLDEN_BIG = ["k40c_%s_%d%d" % (p, a, b) for p in bi.PRECISIONS for a, b in bi.TRANSPOSES] + \
             ["b200_%s_%d%d" % (p, a, b) for p in bi.PRECISIONS for a, b in bi.TRANSPOSES] + \
             ["widened%d_%s_D_00" % (w, d) for w in (64, 256, 512) for d in ("k40c", "b200")] + \
             ["b200_48k_D_00", "b200_48k_S_00"] + \
             ["maxbound_k40c_D_00", "maxbound_k40c_Z_11", "maxbound_b200_D_00"] + \
             sorted(bi.EXTREME)


@pytest.mark.parametrize("key", GOLDEN_BIG)
def test_full_size_vs_golden(beast, golden_expected, key):
    if key not in golden_expected:
        pytest.skip("golden not generated for " + key)
    e = golden_expected[key]
    import torch
    with beast.Space.from_desc(e["space"]) as sp:
        rec, st = sp.enumerate(stats=True)
        assert st["survivors"] == e["survivors"]
        assert st["visits"] == e["visits"], key
        assert st["rejected"] == e["rejected"], key
        assert "0x%016x" % beast.beast_digest(rec) == e["digest"], key
        _check_evaluated(e["space"], st, exact=False)
        if e["first"]:
            lo, hi = rec[0].cpu().numpy(), rec[-1].cpu().numpy()
            assert ["%016x" % lo[1], "%016x" % lo[0]] == e["first"]
            assert ["%016x" % hi[1], "%016x" % hi[0]] == e["last"]
        # strictly increasing as u128 (canonical and unique), on the device
        if len(rec) > 1:
            a = rec.view(torch.int64)
            hi_, lo_ = a[:, 1], a[:, 0]
            # unsigned compare via sign flip
            f = torch.tensor(-(1 << 63), dtype=torch.int64, device=a.device)
            h0, h1 = hi_[:-1] ^ f, hi_[1:] ^ f
            l0, l1 = lo_[:-1] ^ f, lo_[1:] ^ f
            inc = (h0 < h1) | ((h0 == h1) & (l0 < l1))
            assert bool(inc.all())
        # sampled records satisfy all 12 predicates (oracle's evaluator)
        idx = random.Random(1).sample(range(len(rec)), min(300, len(rec)))
        host = rec.view(torch.int64)[idx].cpu().numpy().view(np.uint64) if idx else []
        for lo_v, hi_v in host:
            _, pred = oracle.point(e["space"], oracle.unpack(int(hi_v), int(lo_v)))
            assert not any(pred.values())
        assert sp.count() == e["survivors"]


@pytest.mark.parametrize("world", [2, 3, 8])
def test_virtual_ranks_concatenate(beast, world):
    """Shards (rank, world) concatenated in rank order equal the world=1 list;
    their stats sum to the whole space's."""
    desc = bi.headline()
    full, stf, _, _ = _run(beast, desc)
    parts, visits, rejected = [], np.zeros(15, np.int64), np.zeros(12, np.int64)
    for r in range(world):
        got, st, _, _ = _run(beast, desc, rank=r, world=world)
        parts.append(got)
        visits += np.array(st["visits"], np.int64)
        rejected += np.array(st["rejected"], np.int64)
    cat = np.concatenate(parts)
    assert np.array_equal(cat, full)
    assert list(visits) == stf["visits"] and list(rejected) == stf["rejected"]


def test_digest_is_additive_over_shards(beast):
    import torch
    desc = bi.tiny("C")
    with beast.Space.from_desc(desc) as sp:
        rec = sp.enumerate()
        full = beast.beast_digest(rec)
        k = 1000
        assert (beast.beast_digest(rec[:k]) + beast.beast_digest(rec[k:].contiguous(), base=k)) % (1 << 64) == full
        host = rec.cpu().numpy()
        assert full == oracle.digest(np.stack([host[:, 1], host[:, 0]], 1))
        del torch


def test_capacity_error_reports_required(beast):
    import torch
    with beast.Space.from_desc(bi.tiny("D")) as sp:
        small = torch.empty((10, 2), dtype=torch.uint64, device="cuda")
        with pytest.raises(beast.BeastError) as e:
            beast.beast_enumerate(sp.handle, small)
        assert e.value.status == beast.BEAST_ERR_CAPACITY and "1824" in str(e.value)


def test_enumerate_to_host_matches_device(beast):
    import torch
    desc = bi.headline()
    with beast.Space.from_desc(desc) as sp:
        dev = sp.enumerate().cpu().numpy()
        host = torch.empty((dev.shape[0], 2), dtype=torch.uint64).pin_memory()
        n = beast.beast_enumerate_to_host(sp.handle, host)
        assert n == dev.shape[0]
        assert np.array_equal(host.numpy(), dev)


def test_stats_mode_does_not_change_results(beast):
    desc = bi.k40c("Z")
    with beast.Space.from_desc(desc) as sp:
        a = sp.enumerate().cpu().numpy()
        b, _ = sp.enumerate(stats=True)
        assert np.array_equal(a, b.cpu().numpy())


def test_repeated_calls_are_deterministic(beast):
    desc = bi.headline()
    with beast.Space.from_desc(desc) as sp:
        a = beast.beast_digest(sp.enumerate())
        for _ in range(3):
            assert beast.beast_digest(sp.enumerate()) == a


def test_limits_from_device_b200(beast):
    lim = beast.beast_limits_from_device(0)
    assert lim.cuda_major == 10 and lim.cuda_minor == 0
    for k in ("max_threads_per_block", "max_threads_dim_x", "max_threads_dim_y", "warp_size",
              "max_regs_per_block", "max_registers_per_multi_processor", "float_size",
              "max_shared_mem_per_block", "max_shmem_per_multi_processor"):
        assert getattr(lim, k) == bi.B200_DEVICE[k], (k, getattr(lim, k))
    assert lim.max_blocks_per_multi_processor == 32 and lim.max_registers_per_thread == 255


@pytest.mark.parametrize("key", ["tiny_D_00", "tiny_S_01", "tiny_C_10", "tiny_Z_11", "micro_C_00", "k40c_D_00",
                                 "k40c_S_10", "k40c_C_01", "k40c_Z_11", "b200_D_00", "b200_C_11"])
def test_factorized_equals_canonical(beast, golden_expected, key):
    """the divisor-factorised path gives the same count
    and the same canonical list (digest) as the per-point path / the oracle."""
    e = golden_expected[key]
    with beast.Space.from_desc(e["space"]) as sp:
        assert sp.count_factorized() == e["survivors"]
        rec = sp.enumerate_factorized()
        assert len(rec) == e["survivors"]
        if len(rec):
            assert "0x%016x" % beast.beast_digest(rec) == e["digest"]


@pytest.mark.parametrize("seed", range(0, 200, 7))
def test_factorized_fuzz(beast, seed):
    desc = bi.fuzz_space(seed)
    ref = oracle.nest(desc, records=True)
    with beast.Space.from_desc(desc) as sp:
        rec = sp.enumerate_factorized().cpu().numpy()
    assert np.array_equal(rec, _oracle_lohi(ref["records"]))


def test_factorized_shards(beast):
    desc = bi.headline()
    with beast.Space.from_desc(desc) as sp:
        full = sp.enumerate_factorized().cpu().numpy()
        parts = [sp.enumerate_factorized(rank=r, world=3).cpu().numpy() for r in range(3)]
    assert np.array_equal(np.concatenate(parts), full)


@pytest.mark.gpu
def test_async_passes_match_sync(beast, golden_expected):
    """beast_enumerate_async replays the captured pass; several in flight,
    then beast_wait: same records as the synchronous call."""
    import torch
    e = golden_expected["k40c_D_00"]          # the headline space
    with beast.Space.from_desc(bi.headline()) as sp:
        out = torch.empty((e["survivors"], 2), dtype=torch.uint64, device="cuda")
        with pytest.raises(beast.BeastError):
            beast.beast_enumerate_async(sp.handle, out)          # nothing captured yet
        n = beast.beast_enumerate(sp.handle, out)
        ref = out.clone()
        out.zero_()
        for _ in range(3):
            beast.beast_enumerate_async(sp.handle, out)
        assert beast.beast_wait(sp.handle) == n == e["survivors"]
        torch.cuda.synchronize()
        assert torch.equal(out, ref)
        assert "0x%016x" % beast.beast_digest(out) == e["digest"]
        # a synchronous call after async ones stays in step
        assert beast.beast_enumerate(sp.handle, out) == n


@pytest.mark.gpu
def test_host_async_pipelined_handles(beast, golden_expected):
    """beast_enumerate_to_host_async on two handles, alternating (pass of one
    overlapping the other's host copy): every host list equals the golden
    digest; errors before a synchronous host call and on short capacity."""
    import torch
    e = golden_expected["k40c_D_00"]          # the headline space
    n = e["survivors"]
    sps = [beast.Space.from_desc(bi.headline()) for _ in range(2)]
    try:
        hosts = [torch.empty((n, 2), dtype=torch.uint64).pin_memory() for _ in range(2)]
        streams = [torch.cuda.Stream() for _ in range(2)]
        with pytest.raises(beast.BeastError):
            beast.beast_enumerate_to_host_async(sps[0].handle, hosts[0], stream=streams[0])
        for sp, h, st in zip(sps, hosts, streams):
            assert beast.beast_enumerate_to_host(sp.handle, h, stream=st) == n
        with pytest.raises(beast.BeastError):
            beast.beast_enumerate_to_host_async(sps[0].handle, hosts[0][: n - 1], stream=streams[0])
        with pytest.raises(beast.BeastError):
            beast.beast_enumerate_to_host_async(sps[0].handle, hosts[0], rank=0, world=2, stream=streams[0])
        for i in range(6):
            k = i % 2
            if i >= 2:
                assert beast.beast_wait(sps[k].handle, streams[k]) == n
                dev = hosts[k].cuda()
                assert "0x%016x" % beast.beast_digest(dev) == e["digest"]
            hosts[k].zero_()
            beast.beast_enumerate_to_host_async(sps[k].handle, hosts[k], stream=streams[k])
        for k in range(2):
            assert beast.beast_wait(sps[k].handle, streams[k]) == n
            assert "0x%016x" % beast.beast_digest(hosts[k].cuda()) == e["digest"]
    finally:
        for sp in sps:
            sp.close()


@pytest.mark.gpu
def test_host_async_shards_concatenate(beast, golden_expected):
    """beast_enumerate_to_host_async on shard handles (virtual ranks of 3):
    the host lists concatenated in rank order are the world-1 list."""
    import torch
    e = golden_expected["k40c_D_00"]
    world = 3
    sps = [beast.Space.from_desc(bi.headline()) for _ in range(world)]
    try:
        hosts, streams = [], []
        for r, sp in enumerate(sps):
            n = sp.count(rank=r, world=world)
            hosts.append(torch.empty((n, 2), dtype=torch.uint64).pin_memory())
            streams.append(torch.cuda.Stream())
            assert beast.beast_enumerate_to_host(sp.handle, hosts[r], r, world, streams[r]) == n
            hosts[r].zero_()
        for r, sp in enumerate(sps):
            beast.beast_enumerate_to_host_async(sp.handle, hosts[r], r, world, streams[r])
        for r, sp in enumerate(sps):
            assert beast.beast_wait(sp.handle, streams[r]) == hosts[r].shape[0]
        full = torch.cat(hosts).cuda()
        assert full.shape[0] == e["survivors"]
        assert "0x%016x" % beast.beast_digest(full) == e["digest"]
    finally:
        for sp in sps:
            sp.close()


@pytest.mark.gpu
@pytest.mark.parametrize("seed", range(24))
def test_fuzz_shards_vs_oracle(beast, seed):
    """Shard rule on fuzz spaces: for a seeded world in 2..9
    -- often more ranks than L4 survivors, so some shards are empty -- the
    shards concatenated in rank order are the oracle's list and their
    statistics sum to the oracle's."""
    desc = bi.fuzz_space(seed)
    world = 2 + random.Random(1000 + seed).randrange(8)
    ref = oracle.nest(desc, records=True)
    parts, visits, rejected, counts = [], np.zeros(15, np.int64), np.zeros(12, np.int64), 0
    for r in range(world):
        got, st, _, n = _run(beast, desc, rank=r, world=world)
        assert n == len(got)
        parts.append(got)
        counts += n
        visits += np.array(st["visits"], np.int64)
        rejected += np.array(st["rejected"], np.int64)
    cat = np.concatenate(parts) if parts else np.zeros((0, 2), np.uint64)
    want = _oracle_lohi(ref["records"])
    assert cat.shape == want.shape and np.array_equal(cat, want), (seed, world)
    assert counts == ref["survivors"]
    assert list(visits) == ref["visits"] and list(rejected) == ref["rejected"], (seed, world)

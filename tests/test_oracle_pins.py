"""Pins of the ORACLE against things other than itself (DESIGN.md "Oracle
pins" P1-P8).  CPU only.

P1 brute force            full dependent-range product, every predicate on
                          every point, no early exit (oracle_brute)
P2 invariants             survivors pass all 12 predicates, rejected sampled
                          points fail one, strict u128 order, x16, visit
                          reconciliation
P3 occupancy              Fig 12 occupancy vs the CUDA occupancy-calculator
                          formula on aligned shapes
P4 symmetry               NN <-> TT bijection, ZGEMM transpose invariance
P5 analytic counter       divisor-based counter (oracle/analytic.py)
P6 closed-form N_space    (oracle/closed_form.py) vs the brute force's count
P7 literal transcription  Figs 11-15 as printed, run by a generic evaluator
P8 hand-checked points    tests/golden/worked_points.json
plus the independently produced survey values.
"""
from __future__ import annotations

import json
import os
import random

import numpy as np
import pytest

import beast_inputs as bi
import oracle
import oracle.analytic
import oracle.closed_form
import oracle.literal

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")

# canonical evaluation order of the predicates (level by level, Fig 13 -> 14
# -> 15 within a level; reading A6): L2: 0, 7; L4: 1, 2, 4; L5: 3, 5; L6: 6;
# L9: 8, 10; L11: 9, 11
EVAL_ORDER = (0, 7, 1, 2, 4, 3, 5, 6, 8, 10, 9, 11)


def _load(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def _u128(rec):
    return [(int(h) << 64) | int(l) for h, l in rec]


# ------------------------------------------------------------------ P1, P6
def test_brute_force_micro_c_equals_nest():
    sp = bi.micro("C")
    b = oracle.brute(sp, threads=os.cpu_count())
    n = oracle.nest(sp, records=True)
    assert b["n_space"] == oracle.closed_form.n_space(sp) == 49_499_328
    assert b["survivors"] == n["survivors"] == 64
    assert np.array_equal(b["records"], n["records"])


@pytest.mark.parametrize("seed", range(1000, 1012))
def test_brute_force_fuzz_equals_nest(seed):
    sp = bi.fuzz_space(seed, max_bound=7)
    b = oracle.brute(sp, threads=os.cpu_count())
    n = oracle.nest(sp, records=True)
    assert b["n_space"] == oracle.closed_form.n_space(sp)
    assert b["survivors"] == n["survivors"]
    assert np.array_equal(b["records"], n["records"])


@pytest.mark.slow
def test_brute_force_tiny_dgemm():
    """8,259,231,744 points (P6) -> 1,824 survivors, the brute force keeps
    exactly the nest's list."""
    sp = bi.tiny("D")
    b = oracle.brute(sp, threads=os.cpu_count())
    n = oracle.nest(sp, records=True)
    assert b["n_space"] == oracle.closed_form.n_space(sp) == 8_259_231_744
    assert np.array_equal(b["records"], n["records"])


def test_closed_form_headline():
    assert oracle.closed_form.n_space(bi.headline()) == 136_423_918_516_708_320_149_504


# ---------------------------------------------------------------------- P2
def _check_invariants(sp, r, sample=None, seed=0):
    rec = r["records"]
    assert r["survivors"] % 16 == 0                      # reading A8
    keys = _u128(rec)
    assert all(a < b for a, b in zip(keys, keys[1:]))    # canonical + unique
    idx = range(len(rec)) if sample is None else random.Random(seed).sample(
        range(len(rec)), min(sample, len(rec)))
    for i in idx:
        v = oracle.unpack(*rec[i])
        _, pred = oracle.point(sp, v)
        assert not any(pred.values()), (v, pred)
    V, R = r["visits"], r["rejected"]
    s = oracle.resolve(sp)
    assert V[1] == V[0] * s["dim_n_max"]
    pairs_ok = V[1] - R[0] - R[7]
    assert (pairs_ok == 0) == (V[2] == 0)
    l4_ok = V[3] - R[1] - R[2] - R[4]
    assert V[4] == l4_ok * s["blk_k_max"]
    ndv = 1 if sp["precision"] == "Z" else 2
    assert V[5] == (V[4] - R[3] - R[5]) * ndv
    tuples = V[10] - R[9] - R[11]
    assert V[11] == 2 * tuples and V[12] == 2 * V[11] and V[13] == 2 * V[12] and V[14] == 2 * V[13]
    assert V[14] == r["survivors"]


@pytest.mark.parametrize("p", bi.PRECISIONS)
@pytest.mark.parametrize("ta,tb", bi.TRANSPOSES)
def test_invariants_tiny(p, ta, tb):
    sp = bi.tiny(p, ta, tb)
    _check_invariants(sp, oracle.nest(sp, records=True))


def test_invariants_headline_sampled():
    sp = bi.headline()
    _check_invariants(sp, oracle.nest(sp, threads=os.cpu_count(), records=True), sample=3000)


def _random_point(r, s, dvs):
    dm = r.randint(1, s["dim_m_max"]); dn = r.randint(1, s["dim_n_max"])
    bm = dm * r.randint(1, max(1, s["blk_m_max"] // dm))
    bn = dn * r.randint(1, max(1, s["blk_n_max"] // dn))
    bk = r.randint(1, s["blk_k_max"])
    dv = r.choice(dvs)
    vm = 0 if dv == 1 else r.randint(0, 1)
    ram = (bm if s["trans_a"] == 0 else bk) // dv
    ran = bk if s["trans_a"] == 0 else bm
    rbm = (bk if s["trans_b"] == 0 else bn) // dv
    rbn = bn if s["trans_b"] == 0 else bk
    if min(ram, rbm) < 1 or bm > s["blk_m_max"] or bn > s["blk_n_max"]:
        return None
    return (dm, dn, bm, bn, bk, dv, vm, r.randint(1, ram), r.randint(1, ran),
            r.randint(1, rbm), r.randint(1, rbn), r.randint(0, 1), r.randint(0, 1),
            r.randint(0, 1), r.randint(0, 1))


@pytest.mark.parametrize("p", bi.PRECISIONS)
def test_membership_equals_all_predicates_false(p):
    """A point is in the nest's list iff all 12 predicates are False on it
    (every rejected point violates at least one).  Random points of the
    tiny space, plus near-survivors (a survivor with one coordinate moved)."""
    sp = bi.tiny(p)
    s = oracle.resolve(sp)
    r = oracle.nest(sp, records=True)
    members = set(_u128(r["records"]))
    dvs = (1, 2) if p in ("D", "C") else (1, 4) if p == "S" else (1,)
    rnd = random.Random(7)
    pts = []
    while len(pts) < 3000:
        v = _random_point(rnd, s, dvs)
        if v is not None:
            pts.append(v)
    for h, l in r["records"][:: max(1, len(r["records"]) // 200)]:
        v = list(oracle.unpack(h, l))
        k = rnd.randrange(7, 11)
        v[k] = max(1, v[k] + rnd.choice((-1, 1)))
        pts.append(tuple(v))
    for v in pts:
        _, pred = oracle.point(sp, v)
        key = _u128([_pack(v)])[0]
        assert (key in members) == (not any(pred.values())), v


def _pack(v):
    hi = (v[0] << 52) | (v[1] << 40) | (v[2] << 28) | (v[3] << 16) | (v[4] << 4) | (v[5] << 1) | v[6]
    lo = (v[7] << 52) | (v[8] << 40) | (v[9] << 28) | (v[10] << 16) | (v[11] << 3) | (v[12] << 2) | (v[13] << 1) | v[14]
    return hi, lo


# ---------------------------------------------------------------------- P3
def _cuda_blocks_by_regs(regs_per_thread, threads, regs_sm=65536, unit=256, max_blocks=16):
    """CUDA occupancy calculator, cc 3.5: registers allocated per warp in
    units of 256, warps per block = ceil(threads / 32)."""
    per_warp = -(-regs_per_thread * 32 // unit) * unit
    warps = -(-threads // 32)
    return min((regs_sm // per_warp) // warps, max_blocks)


def _cuda_blocks_by_shmem(smem, smem_sm=49152, unit=256, max_blocks=16):
    return min(smem_sm // (-(-smem // unit) * unit), max_blocks)


@pytest.mark.parametrize("dm,dn,thr_m,thr_n", [
    (16, 16, 4, 4),    # T=256, rpt=32 (double): 8 blocks -> 2048 threads
    (16, 8, 8, 4),     # T=128, rpt=64: 8 blocks
    (32, 32, 2, 2),    # T=1024, rpt=8: 8 blocks
    (8, 4, 2, 2),      # T=32, rpt=8: clamp at 16
    (32, 2, 4, 8),     # T=64, rpt=64: 16 blocks
    (32, 4, 8, 4),     # T=128, rpt=64
    (4, 32, 2, 6),     # T=128, rpt=24
])
def test_occupancy_matches_cuda_calculator_on_aligned_shapes(dm, dn, thr_m, thr_n):
    sp = bi.headline()
    for bk in (1, 8, 16, 32):
        v = (dm, dn, dm * thr_m, dn * thr_n, bk, 1, 0, 1, 1, 1, 1, 0, 0, 0, 0)
        der, _ = oracle.point(sp, v)
        rpt = thr_m * thr_n * 2
        assert rpt % 8 == 0 and (dm * dn) % 32 == 0
        assert der["max_blocks_by_regs"] == _cuda_blocks_by_regs(rpt, dm * dn)
        if der["shmem_per_block"] % 256 == 0:
            assert der["max_blocks_by_shmem"] == _cuda_blocks_by_shmem(der["shmem_per_block"])


def test_occupancy_known_values():
    sp = bi.headline()
    # spb = 16384 -> 3 blocks; spb = 24576 -> 2 blocks (49152 B per SM)
    der, _ = oracle.point(sp, (16, 16, 64, 64, 16, 1, 0, 1, 1, 1, 1, 0, 0, 0, 0))
    assert der["shmem_per_block"] == 16384 and der["max_blocks_by_shmem"] == 3
    der, _ = oracle.point(sp, (16, 16, 64, 128, 16, 1, 0, 1, 1, 1, 1, 0, 0, 0, 0))
    assert der["shmem_per_block"] == 24576 and der["max_blocks_by_shmem"] == 2
    # T=32, rpt=2 (single): min(65536/64, 16) = 16 blocks, as the calculator's
    # block limit
    der, _ = oracle.point(bi.k40c("S"), (32, 1, 32, 1, 1, 1, 0, 1, 1, 1, 1, 0, 0, 0, 0))
    assert der["regs_per_thread"] == 1 and der["max_blocks_by_regs"] == 16
    assert der["max_threads_by_regs"] == 512


# ---------------------------------------------------------------------- P4
def _swap_mn(v):
    dm, dn, bm, bn, bk, dv, vm, dma, dna, dmb, dnb, ta, tb, l1, bk_ = v
    return (dn, dm, bn, bm, bk, dv, vm, dmb, dnb, dma, dna, tb, ta, l1, bk_)


@pytest.mark.parametrize("p", bi.PRECISIONS)
def test_symmetry_nn_tt_bijection_tiny(p):
    nn = oracle.nest(bi.tiny(p, 0, 0), records=True)["records"]
    tt = oracle.nest(bi.tiny(p, 1, 1), records=True)["records"]
    mapped = sorted(_u128([_pack(_swap_mn(oracle.unpack(h, l))) for h, l in nn]))
    assert mapped == _u128(tt)


def test_symmetry_nn_tt_headline_counts():
    a = oracle.nest(bi.headline(0, 0), threads=os.cpu_count(), digest=False)
    b = oracle.nest(bi.headline(1, 1), threads=os.cpu_count(), digest=False)
    assert a["survivors"] == b["survivors"]


def test_zgemm_transpose_invariance_tiny():
    """dim_vec == 1 only: swapping (dim_m_a, dim_n_a) maps trans_a=0 onto
    trans_a=1 (and likewise for B)."""
    base = oracle.nest(bi.tiny("Z", 0, 0), records=True)["records"]
    for ta, tb in bi.TRANSPOSES[1:]:
        other = oracle.nest(bi.tiny("Z", ta, tb), records=True)["records"]
        mapped = []
        for h, l in base:
            v = list(oracle.unpack(h, l))
            if ta:
                v[7], v[8] = v[8], v[7]
            if tb:
                v[9], v[10] = v[10], v[9]
            mapped.append(_pack(v))
        assert sorted(_u128(mapped)) == _u128(other)


# ---------------------------------------------------------------------- P5
@pytest.mark.parametrize("p", bi.PRECISIONS)
@pytest.mark.parametrize("ta,tb", bi.TRANSPOSES)
def test_analytic_equals_nest_tiny(p, ta, tb):
    sp = bi.tiny(p, ta, tb)
    a = oracle.analytic.count(sp)
    n = oracle.nest(sp)
    assert a["visits"] == n["visits"] and a["rejected"] == n["rejected"]


@pytest.mark.parametrize("seed", range(20))
def test_analytic_equals_nest_fuzz(seed):
    sp = bi.fuzz_space(seed)
    a = oracle.analytic.count(sp)
    n = oracle.nest(sp)
    assert a["visits"] == n["visits"] and a["rejected"] == n["rejected"]


@pytest.mark.parametrize("ta,tb", bi.TRANSPOSES)
def test_analytic_equals_nest_dgemm_k40c(ta, tb):
    sp = bi.headline(ta, tb)
    a = oracle.analytic.count(sp)
    n = oracle.nest(sp, threads=os.cpu_count(), digest=False)
    assert a["visits"] == n["visits"] and a["rejected"] == n["rejected"]


# ---------------------------------------------------------------------- P7
@pytest.mark.parametrize("p", bi.PRECISIONS)
@pytest.mark.parametrize("ta,tb", bi.TRANSPOSES)
def test_literal_transcription_equals_nest_tiny(p, ta, tb):
    sp = bi.tiny(p, ta, tb)
    lit = oracle.literal.run(sp, oracle.resolve(sp))
    n = oracle.nest(sp, records=True)
    assert lit["visits"] == n["visits"]
    assert lit["rejected"] == n["rejected"]
    assert sorted(_u128([_pack(v) for v in lit["records"]])) == _u128(n["records"])
    assert [_pack(v) for v in lit["records"]] == [(int(h), int(l)) for h, l in n["records"]]


@pytest.mark.parametrize("seed", range(8))
def test_literal_transcription_equals_nest_fuzz(seed):
    sp = bi.fuzz_space(seed, max_bound=12)
    lit = oracle.literal.run(sp, oracle.resolve(sp))
    n = oracle.nest(sp)
    assert lit["visits"] == n["visits"] and lit["rejected"] == n["rejected"]


# ---------------------------------------------------------------------- P8
def test_worked_survivor_point():
    g = _load("worked_points.json")
    sp = bi.tiny("D")
    der, pred = oracle.point(sp, g["survivor"]["tuple"])
    assert der == g["survivor"]["derived"]
    assert not any(pred.values())
    rec = oracle.nest(sp, records=True)["records"]
    assert _u128([_pack(g["survivor"]["tuple"])])[0] in set(_u128(rec))


def test_worked_rejected_points():
    g = _load("worked_points.json")
    sp = bi.headline()
    for case in g["rejected"]:
        _, pred = oracle.point(sp, case["tuple"])
        vals = list(pred.values())
        first = next(oracle.PREDICATES[i] for i in EVAL_ORDER if vals[i])
        assert first == case["first_failing"], case


# ------------------------------------------------- survey values (external)
def test_survey_appendix_tiny_and_headline():
    g = _load("survey_appendix_a.json")
    r = oracle.nest(bi.tiny("D"))
    assert r["visits"] == g["tiny_d_nn_visits"]
    want = dict.fromkeys(oracle.PREDICATES, 0)
    want.update(g["tiny_d_nn_rejected"])
    assert r["rejected"] == [want[k] for k in oracle.PREDICATES]
    for p in bi.PRECISIONS:
        for ta, tb in bi.TRANSPOSES:
            assert oracle.nest(bi.tiny(p, ta, tb))["survivors"] == g["tiny"]["survivors"][p]
        assert sum(oracle.nest(bi.tiny(p))["visits"]) == g["tiny"]["n_canon_nn"][p]
    h = oracle.nest(bi.headline(), threads=os.cpu_count())
    assert h["visits"] == g["headline_visits"]
    assert h["rejected"] == [g["headline_rejected"][k] for k in oracle.PREDICATES]


def test_survey_appendix_digests_small():
    g = _load("survey_appendix_a.json")
    spaces = {"tiny D NN K40c": bi.tiny("D"), "tiny S NN K40c": bi.tiny("S"),
              "tiny Z NN K40c": bi.tiny("Z"), "tiny C NN K40c": bi.tiny("C"),
              "micro C NN K40c": bi.micro("C"), "headline D NN K40c": bi.headline(),
              "D TN K40c": bi.headline(1, 0), "D NT K40c": bi.headline(0, 1),
              "D TT K40c": bi.headline(1, 1), "Z NN K40c": bi.k40c("Z")}
    for d in g["digests"]:
        if d["space"] not in spaces:
            continue
        r = oracle.nest(spaces[d["space"]], threads=os.cpu_count(), records=True)
        assert r["survivors"] == d["survivors"]
        assert "0x%016x" % r["digest"] == d["digest"]
        assert ["%016x" % x for x in r["records"][0]] == d["first"]
        assert ["%016x" % x for x in r["records"][-1]] == d["last"]
        assert oracle.digest(r["records"]) == r["digest"]


def test_survey_appendix_k40c_table_from_golden(golden_expected):
    """expected.json (written by scripts/make_golden.py from the oracle) agrees
    with the survey's independently computed K40c / B200 tables."""
    g = _load("survey_appendix_a.json")
    for dev in ("k40c", "b200"):
        for p, rows in g[dev].items():
            for (ta, tb), (surv, ncanon) in zip(bi.TRANSPOSES, rows):
                key = "%s_%s_%d%d" % (dev, p, ta, tb)
                if key not in golden_expected:
                    continue
                e = golden_expected[key]
                assert (e["survivors"], e["n_canon"]) == (surv, ncanon), key
    for d in g["digests"]:
        key = {"S NN K40c": "k40c_S_00", "C NN K40c": "k40c_C_00", "D NN B200": "b200_D_00"}.get(d["space"])
        if key and key in golden_expected:
            e = golden_expected[key]
            assert e["digest"] == d["digest"] and e["survivors"] == d["survivors"]
            if e["first"]:
                assert e["first"] == d["first"] and e["last"] == d["last"]
    for b, vals in g["widened_dgemm_nn"].items():
        for dev, (surv, ncanon) in vals.items():
            key = "widened%s_%s_D_00" % (b, dev)
            if key in golden_expected:
                assert (golden_expected[key]["survivors"], golden_expected[key]["n_canon"]) == (surv, ncanon)
    if "b200_S_00" in golden_expected:
        e = golden_expected["b200_S_00"]
        assert e["visits"] == g["sgemm_b200_visits"]
        assert e["rejected"] == [g["sgemm_b200_rejected"][k] for k in oracle.PREDICATES]
        assert e["valid_a"] == g["sgemm_b200_frontier"]["valid_a"]
    for k, (surv, ncanon) in g["b200_48k"].items():
        key = "b200_48k_%s_00" % k
        if key in golden_expected:
            assert (golden_expected[key]["survivors"], golden_expected[key]["n_canon"]) == (surv, ncanon)


def test_golden_expected_matches_nest_small(golden_expected):
    """The stored expectations are the oracle's current output."""
    for key in ("tiny_D_00", "tiny_C_11", "micro_C_00", "k40c_Z_10"):
        e = golden_expected[key]
        r = oracle.nest(e["space"], threads=os.cpu_count())
        assert r["survivors"] == e["survivors"] and r["visits"] == e["visits"]
        assert "0x%016x" % r["digest"] == e["digest"]


def test_digest_definition():
    """SURVEY §8(b) digest, restated: order-sensitive through the index and
    additive over shards."""
    rec = oracle.nest(bi.tiny("C"), records=True)["records"]
    full = oracle.digest(rec)
    k = 1000
    assert (oracle.digest(rec[:k]) + oracle.digest(rec[k:], base=k)) % (1 << 64) == full
    swapped = rec.copy()
    swapped[[3, 4]] = swapped[[4, 3]]
    assert oracle.digest(swapped) != full


def test_fig9_lookup():
    # Fig 9: K40c cc 3.5 -> 16 blocks, 64 warps, 255 regs;
    # cc 2.x -> 8, 48, 63; cc 1.3 -> 8, 32, 128; unused entries -1; A10 cc 10.0
    assert [oracle.fig9_lookup(3, 5, w) for w in range(3)] == [16, 64, 255]
    assert [oracle.fig9_lookup(2, 1, w) for w in range(3)] == [8, 48, 63]
    assert [oracle.fig9_lookup(1, 3, w) for w in range(3)] == [8, 32, 128]
    assert oracle.fig9_lookup(3, 2, 0) == -1
    assert [oracle.fig9_lookup(10, 0, w) for w in range(3)] == [32, 64, 255]

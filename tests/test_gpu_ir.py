"""GPU parity of the generic space IR engine:
NVRTC-compiled level-wise enumeration (csrc/beast_ir.cu) against

* the IR oracle (oracle/ir.py: the same description as plain C nested
  loops) and the by-definition brute force, on the toy specs;
* the hand-written canonical GEMM nest (oracle.nest) on the paper's GEMM
  space written in the IR (tests/ir_specs.gemm_spec): full survivor list in
  canonical order, per-level visits, first-failing rejections.

Integer work: bit-exact.
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
from test_ir_oracle import pack  # noqa: E402

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


@pytest.mark.parametrize("name", sorted(ir_specs.toy_specs()))
def test_toy_specs(beast, name):
    spec = ir_specs.toy_specs()[name]
    ref = oir.run(spec, records=True)
    with beast.IRSpace(spec) as sp:
        rec, st = sp.enumerate()
        cnt = sp.count()
    assert st == cnt
    assert st["survivors"] == ref["survivors"] == len(ir_specs.brute(spec))
    assert st["visits"] == ref["visits"] and st["rejected"] == ref["rejected"]
    assert np.array_equal(rec.cpu().numpy(), ref["records"])


def _gemm(beast, desc):
    spec = ir_specs.gemm_spec(oracle.resolve(desc), desc["precision"])
    ref = oracle.nest(desc, records=True)
    with beast.IRSpace(spec) as sp:
        rec, st = sp.enumerate()
    assert st["survivors"] == ref["survivors"]
    assert st["visits"] == ref["visits"]
    assert st["rejected"] == ref["rejected"]
    assert np.array_equal(pack(rec.cpu().numpy()), ref["records"].astype(np.uint64))


@pytest.mark.parametrize("p", bi.PRECISIONS)
@pytest.mark.parametrize("ta,tb", bi.TRANSPOSES)
def test_gemm_ir_tiny(beast, p, ta, tb):
    _gemm(beast, bi.tiny(p, ta, tb))


@pytest.mark.parametrize("seed", range(6))
def test_gemm_ir_fuzz(beast, seed):
    _gemm(beast, bi.fuzz_space(seed))


def test_gemm_ir_medium_against_ir_oracle(beast):
    # K40c DGEMM with all five bounds 48: ~10^8 canonical points
    desc = bi.make_space(bi.K40C_DEVICE, "D", bounds=48)
    spec = ir_specs.gemm_spec(oracle.resolve(desc), "D")
    ref = oir.run(spec, records=True)
    with beast.IRSpace(spec) as sp:
        rec, st = sp.enumerate()
    assert st["survivors"] == ref["survivors"] > 0
    assert st["visits"] == ref["visits"] and st["rejected"] == ref["rejected"]
    assert np.array_equal(rec.cpu().numpy(), ref["records"])
    nest = oracle.nest(desc, records=True)
    assert np.array_equal(pack(rec.cpu().numpy()), nest["records"].astype(np.uint64))


def test_capacity_error(beast):
    import ctypes

    import torch
    spec = ir_specs.toy_specs()["multiples"]
    with beast.IRSpace(spec) as sp:
        n = sp.count()["survivors"]
        out = torch.empty((n - 1, 3), dtype=torch.int64, device="cuda")
        w = ctypes.c_uint64(0)
        rc = beast._lib.lib().beast_ir_enumerate(sp.handle, None, ctypes.c_void_p(out.data_ptr()), n - 1,
                                                 ctypes.byref(w), None, None)
        assert rc == beast.BEAST_ERR_CAPACITY and w.value == n


class _Env:
    """Force the engine's alternative kernel shapes (read by each run): the
    thread-per-parent kernels on every level (BEAST_IR_THREAD_MIN = 0) and/or
    the fused two-level kernels wherever a level has no constraints
    (BEAST_IR_FUSE_MIN = 0: warp per parent; with BEAST_IR_THREAD_MIN = 0:
    thread per parent), or the fusion the engine chooses when a level's rows
    would exceed BEAST_IR_MATERIALIZE_MAX bytes (0: always) -- by default
    they serve only levels with many parents or rows, which the small parity
    spaces never reach."""

    MODES = {"thread": {"BEAST_IR_THREAD_MIN": "0"},
             "fused": {"BEAST_IR_FUSE_MIN": "0"},                  # warp per parent, fused pairs
             "fused_thread": {"BEAST_IR_THREAD_MIN": "0", "BEAST_IR_FUSE_MIN": "0"},
             "adaptive": {"BEAST_IR_MATERIALIZE_MAX": "0"}}        # fuse wherever rows would materialise

    def __init__(self, mode):
        self.vars = self.MODES[mode]

    def __enter__(self):
        self.old = {k: os.environ.get(k) for k in self.vars}
        os.environ.update(self.vars)

    def __exit__(self, *exc):
        for k, v in self.old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


@pytest.mark.parametrize("mode", sorted(_Env.MODES))
@pytest.mark.parametrize("name", sorted(ir_specs.toy_specs()))
def test_toy_specs_kernel_shapes(beast, name, mode):
    with _Env(mode):
        test_toy_specs(beast, name)


@pytest.mark.parametrize("mode", sorted(_Env.MODES))
@pytest.mark.parametrize("p", bi.PRECISIONS)
def test_gemm_ir_tiny_kernel_shapes(beast, p, mode):
    with _Env(mode):
        _gemm(beast, bi.tiny(p, 0, 1))


@pytest.mark.parametrize("mode", sorted(_Env.MODES))
def test_gemm_ir_medium_kernel_shapes(beast, mode):
    with _Env(mode):
        test_gemm_ir_medium_against_ir_oracle(beast)


@pytest.mark.parametrize("which", ["tiny_D", "fuzz_11", "toy"])
def test_replayed_runs_equal_first(beast, which):
    """After its first run a handle enqueues every level without a host
    round trip, sizing each level from the previous run's totals (checked at
    the end): later counts and enumerations must equal the first and the
    oracle's."""
    if which == "toy":
        spec = ir_specs.toy_specs()[sorted(ir_specs.toy_specs())[0]]
        ref = oir.run(spec, records=True)
        want = ref["records"]
    else:
        desc = bi.tiny("D") if which == "tiny_D" else bi.fuzz_space(11)
        spec = ir_specs.gemm_spec(oracle.resolve(desc), desc["precision"])
        ref = oracle.nest(desc, records=True)
        want = None
    with beast.IRSpace(spec) as sp:
        first = sp.count()
        for _ in range(3):
            assert sp.count() == first
            rec, st = sp.enumerate()
            assert st == first
            got = rec.cpu().numpy()
            if want is not None:
                assert np.array_equal(got, want)
            else:
                assert np.array_equal(pack(got), ref["records"].astype(np.uint64))
    assert first["survivors"] == ref["survivors"] and first["visits"] == ref["visits"]

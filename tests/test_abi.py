"""The C-ABI library loads, exports every symbol include/beast.h declares, and
its host-only entry points (limits presets, validation, resolution) behave as
documented.  No compute call: CPU only."""
from __future__ import annotations

import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared_functions():
    src = open(os.path.join(ROOT, "include", "beast.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    names = re.findall(r"\b(beast_[a-z0-9_]+)\s*\(", src)
    return sorted(set(n for n in names if not n.endswith("_fn")))


@pytest.fixture(scope="module")
def beast():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_luszczekgkdd16_b200 as b
    return b


def test_exports_every_declared_symbol(beast):
    from paper_conf_ipps_luszczekgkdd16_b200 import _lib
    L = ctypes.CDLL(_lib.LIB_PATH)
    declared = _declared_functions()
    assert len(declared) >= 15
    for name in declared:
        assert hasattr(L, name), name
    assert set(declared) == set(_lib.EXPORTED)


def test_binding_names_match_abi(beast):
    for name in ("beast_space_create", "beast_space_destroy", "beast_count", "beast_enumerate",
                 "beast_enumerate_to_host", "beast_digest", "beast_limits_k40c",
                 "beast_limits_from_device", "beast_abi_version"):
        assert callable(getattr(beast, name)), name


def test_abi_version(beast):
    import ctypes
    import re
    hdr = open(os.path.join(ROOT, "include", "beast.h")).read()
    assert beast.beast_abi_version() == int(re.search(r"#define BEAST_ABI_VERSION (\d+)", hdr).group(1)) == 2
    # beast_stats: 15 visits + 12 rejections + 4 counts + formed[2] + checked[2] + l4_digest
    assert ctypes.sizeof(beast.beast_stats) == 8 * (15 + 12 + 4 + 2 + 2 + 1)


def test_k40c_preset_is_fig8_and_fig9(beast):
    import beast_inputs
    lim = beast.beast_limits_k40c()
    for k, v in beast_inputs.K40C_DEVICE.items():
        assert getattr(lim, k) == v, k
    # Fig 9 [3][5]
    assert (lim.max_blocks_per_multi_processor, lim.max_warps_per_multi_processor,
            lim.max_registers_per_thread) == (16, 64, 255)


def test_resolution_matches_oracle(beast):
    """The library's Fig 9 table and default bounds resolve every named space
    exactly as the oracle's independent copy does."""
    import beast_inputs
    import oracle
    for name in beast_inputs.NAMED:
        desc = beast_inputs.named(name)
        sp = beast.Space.from_desc(desc, torch_alloc=False)
        got = sp.resolved()
        sp.close()
        want = oracle.resolve(desc)
        for k, v in got.items():
            assert v == want[k], (name, k, v, want[k])


def test_resolution_fuzz(beast):
    import beast_inputs
    import oracle
    for seed in range(50):
        desc = beast_inputs.fuzz_space(seed)
        sp = beast.Space.from_desc(desc, torch_alloc=False)
        got = sp.resolved()
        sp.close()
        want = oracle.resolve(desc)
        assert all(got[k] == want[k] for k in got), seed


def test_validation(beast):
    import beast_inputs
    lim = beast.beast_limits_k40c()
    with pytest.raises(beast.BeastError) as e:
        beast.beast_space_create(lim, "D", None, beast.beast_bounds(4096, 16, 16, 16, 16))
    assert e.value.status == -2
    bad = beast.limits_from_desc(dict(beast_inputs.K40C_DEVICE, warp_size=0))
    with pytest.raises(beast.BeastError):
        beast.beast_space_create(bad, "D")
    nocc = beast.limits_from_desc(dict(beast_inputs.K40C_DEVICE, cuda_major=7, cuda_minor=0))
    with pytest.raises(beast.BeastError) as e:
        beast.beast_space_create(nocc, "D")
    assert e.value.status == -2
    with pytest.raises(beast.BeastError) as e:
        beast.beast_space_create(lim, 7)
    assert e.value.status == -1
    with pytest.raises(beast.BeastError):
        beast.beast_space_create(lim, "D", beast.beast_settings(2, 0, 256, 2))
    h = beast.beast_space_create(lim, "Z", None, None)
    beast.beast_space_destroy(h)


def test_bad_rank_world_rejected_before_device_work(beast):
    h = beast.beast_space_create(beast.beast_limits_k40c(), "D")
    from paper_conf_ipps_luszczekgkdd16_b200 import _lib
    n = ctypes.c_uint64(0)
    assert _lib.lib().beast_count(h, 2, 2, None, ctypes.byref(n), None) == -1
    assert _lib.lib().beast_count(h, 0, 0, None, ctypes.byref(n), None) == -1
    beast.beast_space_destroy(h)


def test_error_strings(beast):
    from paper_conf_ipps_luszczekgkdd16_b200 import _lib
    for code in range(0, -6, -1):
        assert _lib.lib().beast_error_string(code)


def test_product_package_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_ipps_luszczekgkdd16_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                txt = open(os.path.join(dirpath, f)).read()
                assert "oracle" not in re.sub(r"#.*|//.*", "", txt).replace("oracle/", ""), f

"""Seeded, synthetic space descriptions shared by the oracle tests, the GPU
parity tests and bench.py.

This module holds INPUTS only — device-query values, settings, bounds and
thresholds — and none of the method's arithmetic: no Fig 9 lookup, no
derived variable, no predicate.  Both the oracle (oracle/) and the CUDA
library resolve Fig 9 and the Fig 11 default bounds themselves.

A space description is a flat dict whose keys are the field names of
`beast_space_desc` in include/beast.h (and of the oracle's struct):

* Fig 8 device query — the twelve `cudaGetDeviceProperties`
  values, including cuda_major / cuda_minor;
* Fig 9 lookups — max_blocks_per_multi_processor,
  max_warps_per_multi_processor, max_registers_per_thread; 0 means "look up
  from the compute capability", a positive value overrides;
* Fig 10 settings — precision as 'S', 'D', 'C' or 'Z'
  (single/real, double/real, single/complex, double/complex), trans_a, trans_b;
* Fig 14 thresholds;
* Fig 11 upper limits — 0 means the paper default
  (reading A9 in DESIGN.md).
"""
from __future__ import annotations

import random

PRECISIONS = ("S", "D", "C", "Z")
TRANSPOSES = ((0, 0), (1, 0), (0, 1), (1, 1))

# Fig 8: device information of a Tesla K40c.
K40C_DEVICE = dict(
    max_threads_per_block=1024,
    max_threads_dim_x=1024,
    max_threads_dim_y=1024,
    max_shared_mem_per_block=49152,
    warp_size=32,
    max_regs_per_block=65536,
    max_threads_per_multi_processor=2048,
    cuda_major=3,
    cuda_minor=5,
    max_registers_per_multi_processor=65536,
    max_shmem_per_multi_processor=49152,
    float_size=4,
)

# B200 (sm_100) device limits, reading A10 of DESIGN.md: the Fig 8 fields as
# cudaGetDeviceProperties reports them on a B200, with the opt-in 227 KB
# per-block shared memory (sharedMemPerBlockOptin) and 228 KB per SM.
B200_DEVICE = dict(
    max_threads_per_block=1024,
    max_threads_dim_x=1024,
    max_threads_dim_y=1024,
    max_shared_mem_per_block=232448,
    warp_size=32,
    max_regs_per_block=65536,
    max_threads_per_multi_processor=2048,
    cuda_major=10,
    cuda_minor=0,
    max_registers_per_multi_processor=65536,
    max_shmem_per_multi_processor=233472,
    float_size=4,
)

# The 48 KB default per-block variant of the B200 limits (A10, reported
# alongside the opt-in figure).
B200_48K_DEVICE = dict(B200_DEVICE, max_shared_mem_per_block=49152)

FIG9_FIELDS = ("max_blocks_per_multi_processor", "max_warps_per_multi_processor",
               "max_registers_per_thread")
BOUND_FIELDS = ("dim_m_max", "dim_n_max", "blk_m_max", "blk_n_max", "blk_k_max")
DEVICE_FIELDS = tuple(K40C_DEVICE) + FIG9_FIELDS
SETTING_FIELDS = ("precision", "trans_a", "trans_b",
                  "min_threads_per_multi_processor", "min_fmas_per_load")
ALL_FIELDS = DEVICE_FIELDS + SETTING_FIELDS + BOUND_FIELDS


def make_space(device: dict, precision: str = "D", trans_a: int = 0, trans_b: int = 0,
               bounds=None, min_threads_per_multi_processor: int = 256,
               min_fmas_per_load: int = 2, **fig9) -> dict:
    """A full space description.  `bounds` is None (paper defaults), an int
    (all five bounds) or a 5-tuple (dim_m, dim_n, blk_m, blk_n, blk_k)."""
    if precision not in PRECISIONS:
        raise ValueError(precision)
    d = {k: int(device[k]) for k in K40C_DEVICE}
    for k in FIG9_FIELDS:
        d[k] = int(fig9.get(k, device.get(k, 0)))
    d.update(precision=precision, trans_a=int(trans_a), trans_b=int(trans_b),
             min_threads_per_multi_processor=int(min_threads_per_multi_processor),
             min_fmas_per_load=int(min_fmas_per_load))
    if bounds is None:
        b = (0,) * 5
    elif isinstance(bounds, int):
        b = (bounds,) * 5
    else:
        b = tuple(int(x) for x in bounds)
        assert len(b) == 5
    d.update(zip(BOUND_FIELDS, b))
    return d


def tiny(precision="D", trans_a=0, trans_b=0):
    """BASELINE.json configs[0]: K40c limits, all five bounds 16."""
    return make_space(K40C_DEVICE, precision, trans_a, trans_b, bounds=16)


def micro(precision="C", trans_a=0, trans_b=0):
    """Bounds 8, K40c limits (brute-forceable in about a second)."""
    return make_space(K40C_DEVICE, precision, trans_a, trans_b, bounds=8)


def headline(trans_a=0, trans_b=0):
    """BASELINE.json configs[1]: the paper's timed case — DGEMM, no
    transposes, K40c limits, default bounds (PAPER.md:904-907, 1708-1713,
    1976-1981)."""
    return make_space(K40C_DEVICE, "D", trans_a, trans_b)


def k40c(precision, trans_a=0, trans_b=0):
    """BASELINE.json configs[2]: any precision x transpose, K40c limits."""
    return make_space(K40C_DEVICE, precision, trans_a, trans_b)


def b200(precision, trans_a=0, trans_b=0, smem_48k=False):
    """BASELINE.json configs[3]: B200 (sm_100) limits."""
    return make_space(B200_48K_DEVICE if smem_48k else B200_DEVICE, precision, trans_a, trans_b)


def widened(blk_max=256, device="k40c", precision="D", trans_a=0, trans_b=0):
    """BASELINE.json configs[4]: dims up to the device default, blk_m, blk_n,
    blk_k up to `blk_max` (reading A19)."""
    dev = K40C_DEVICE if device == "k40c" else B200_DEVICE
    return make_space(dev, precision, trans_a, trans_b,
                      bounds=(0, 0, blk_max, blk_max, blk_max))


def maxbound(device="k40c", precision="D", trans_a=0, trans_b=0):
    """Edge case: all five iterator bounds at 4095, the largest the packed
    12-bit record fields (and the library's validation) admit."""
    dev = K40C_DEVICE if device == "k40c" else B200_DEVICE
    return make_space(dev, precision, trans_a, trans_b, bounds=4095)


NAMED = {
    "tiny": lambda: tiny("D"),
    "micro": lambda: micro("C"),
    "headline": headline,
    "k40c_S": lambda: k40c("S"),
    "k40c_C": lambda: k40c("C"),
    "k40c_Z": lambda: k40c("Z"),
    "b200_D": lambda: b200("D"),
    "b200_S": lambda: b200("S"),
    "b200_C": lambda: b200("C"),
    "b200_Z": lambda: b200("Z"),
    "widened256_k40c": lambda: widened(256, "k40c"),
    "widened256_b200": lambda: widened(256, "b200"),
}


def named(name: str) -> dict:
    return NAMED[name]()


def _log_int(r: random.Random, lo: int, hi: int) -> int:
    """Integer in [lo, hi], log-uniform (lo >= 1)."""
    import math
    return min(hi, max(lo, int(math.exp(r.uniform(math.log(lo), math.log(hi + 1))))))


# Admitted ranges of beast_space_create (include/beast.h): the widest values
# the library accepts.  fuzz_space_wide draws from these.
ADMITTED = dict(max_threads_per_block=65535, float_size=1024, max_blocks_per_multi_processor=65534,
                min_threads_per_multi_processor=1 << 30, min_fmas_per_load=1 << 20, bound=4095,
                int32=(1 << 31) - 1)


def fuzz_space_wide(seed: int, attempt: int = 0) -> dict:
    """Seeded random space over the library's whole admitted range (seeds
    200-399 of the test plan): max_threads_per_block up to 65535 (so
    threads_per_block up to 65535), warp_size in {1, ..., 64}, every bound up
    to 4095, float_size up to 1024, max_blocks_per_multi_processor up to
    65534, shared-memory / register limits and max_registers_per_thread up
    to 2^31 - 1, thresholds min_threads up to 2^30 and min_fmas up to 2^20.
    Three regimes, so that the draws also leave survivors: "hostile" (every
    value log-uniform over its whole range, the cap one time in five),
    "friendly" (limits drawn from the permissive upper part of their ranges,
    small thresholds) and "big_t" (friendly, with max_threads_per_block >=
    2048 and bounds 16-512, where threads_per_block > 1024 survives).
    `attempt` re-draws the same seed (scripts/make_wide_fuzz.py keeps the
    first attempt whose canonical nest the oracle finishes within its
    budget)."""
    r = random.Random(seed * 7919 + attempt * 104729 + 17)
    A = ADMITTED
    mode = r.choices(("hostile", "friendly", "big_t"), (0.3, 0.3, 0.4))[0]

    def draw(lo, typical, hi):
        """the cap (1/5), log-uniform over [lo, typical] (2/5) or over the
        whole admitted range [lo, hi] (2/5)"""
        u = r.random()
        if u < 0.2:
            return hi
        return _log_int(r, lo, typical if u < 0.6 else hi)

    def high(lo, hi):
        """the cap (1/2) or log-uniform over [lo, hi]"""
        return hi if r.random() < 0.5 else _log_int(r, lo, hi)

    warp = r.choice((1, 2, 4, 8, 16, 32, 64))
    dev = dict(K40C_DEVICE)
    dev["warp_size"] = warp
    dev["float_size"] = draw(1, 16, A["float_size"])
    if mode == "hostile":
        dev["max_threads_per_block"] = draw(warp, 4096, A["max_threads_per_block"])
        dev["max_shared_mem_per_block"] = draw(16, 1 << 18, A["int32"])
        dev["max_shmem_per_multi_processor"] = draw(16, 1 << 18, A["int32"])
        dev["max_regs_per_block"] = draw(1, 1 << 17, A["int32"])
        dev["max_registers_per_multi_processor"] = draw(1, 1 << 17, A["int32"])
        fig9 = dict(max_blocks_per_multi_processor=draw(1, 64, A["max_blocks_per_multi_processor"]),
                    max_registers_per_thread=draw(1, 256, A["int32"]))
        bounds = tuple(draw(1, 128, A["bound"]) for _ in range(5))
        mt = 0 if r.random() < 0.1 else draw(1, 2048, A["min_threads_per_multi_processor"])
        mf = 0 if r.random() < 0.1 else draw(1, 8, A["min_fmas_per_load"])
    elif mode == "friendly":
        dev["max_threads_per_block"] = high(warp, A["max_threads_per_block"])
        dev["max_shared_mem_per_block"] = high(1 << 16, A["int32"])
        dev["max_shmem_per_multi_processor"] = high(1 << 16, A["int32"])
        dev["max_regs_per_block"] = high(1 << 16, A["int32"])
        dev["max_registers_per_multi_processor"] = high(1 << 16, A["int32"])
        fig9 = dict(max_blocks_per_multi_processor=high(8, A["max_blocks_per_multi_processor"]),
                    max_registers_per_thread=high(64, A["int32"]))
        bounds = tuple(draw(1, 128, A["bound"]) for _ in range(5))
        u = r.random()
        mt = 0 if u < 0.2 else A["min_threads_per_multi_processor"] if u < 0.25 else _log_int(r, 1, 2048)
        u = r.random()
        mf = 0 if u < 0.2 else A["min_fmas_per_load"] if u < 0.25 else _log_int(r, 1, 8)
    else:
        # big_t: few resident blocks and a high occupancy threshold keep
        # only large threads_per_block (min_threads / max_blocks), few
        # registers per thread keep blk_m, blk_n near dim_m, dim_n
        dev["max_threads_per_block"] = high(4096, A["max_threads_per_block"])
        for k in ("max_shared_mem_per_block", "max_shmem_per_multi_processor", "max_regs_per_block",
                  "max_registers_per_multi_processor"):
            dev[k] = A["int32"] if r.random() < 0.7 else _log_int(r, 1 << 22, A["int32"])
        mb = r.randint(1, 4)
        fig9 = dict(max_blocks_per_multi_processor=mb, max_registers_per_thread=_log_int(r, 8, 256))
        bounds = (_log_int(r, 64, 1024), _log_int(r, 64, 1024), _log_int(r, 64, 2048),
                  _log_int(r, 64, 2048), _log_int(r, 32, 1024))
        mt = mb * _log_int(r, 1024, max(1024, dev["max_threads_per_block"] // 2))
        mf = r.randint(0, 1)
    fig9["max_warps_per_multi_processor"] = r.choice((16, 32, 48, 64))
    return make_space(dev, r.choice(PRECISIONS), r.randint(0, 1), r.randint(0, 1), bounds=bounds,
                      min_threads_per_multi_processor=mt, min_fmas_per_load=mf, **fig9)


# Edge spaces at the limits beast_space_create admits (include/beast.h):
# threads_per_block up to 65535, float_size 1024, max_blocks 65534 with the
# occupancy threshold 2^30, min_fmas 2^20, limits at 2^31 - 1.  Goldens come
# from scripts/make_golden.py (oracle only).
_INT32 = (1 << 31) - 1
_OPEN = dict(K40C_DEVICE, max_threads_per_block=65535, max_shared_mem_per_block=_INT32,
             max_shmem_per_multi_processor=_INT32, max_regs_per_block=_INT32,
             max_registers_per_multi_processor=_INT32)
EXTREME = {
    # 16384 <= threads_per_block <= 65535, a multiple of 64 (one resident
    # block must reach the occupancy threshold)
    "ext_bigT_D_00": lambda: make_space(dict(_OPEN, warp_size=64), "D", 0, 0, bounds=(256, 256, 512, 512, 256),
                                        min_threads_per_multi_processor=16384, min_fmas_per_load=0,
                                        max_blocks_per_multi_processor=1, max_registers_per_thread=4),
    # threads_per_block >= 4096, any multiple of 1, SGEMM (dim_vec 4), both transposes
    "ext_bigT_S_11": lambda: make_space(dict(_OPEN, warp_size=1), "S", 1, 1, bounds=(128, 128, 256, 256, 64),
                                        min_threads_per_multi_processor=4096, min_fmas_per_load=1,
                                        max_blocks_per_multi_processor=1, max_registers_per_thread=8),
    # float_size 1024 against 2^31 - 1 bytes of shared memory
    "ext_float1024_C_10": lambda: make_space(dict(_OPEN, max_threads_per_block=4096, float_size=1024), "C", 1, 0,
                                             bounds=(64, 64, 128, 128, 128),
                                             max_blocks_per_multi_processor=32, max_registers_per_thread=255),
    # max_blocks 65534 and min_threads 65534 * 32: need = ceil(min_threads / T)
    # is 65534 at T = 32 and exceeds max_blocks below it (the saturated
    # need of the packed L3 row word)
    "ext_need_edge_D_00": lambda: make_space(dict(_OPEN, warp_size=1, float_size=1), "D", 0, 0,
                                             bounds=(64, 64, 128, 128, 64),
                                             min_threads_per_multi_processor=65534 * 32, min_fmas_per_load=0,
                                             max_blocks_per_multi_processor=65534, max_registers_per_thread=255),
    # min_threads 2^30 with max_blocks 65534 (threads_per_block >= 16385 needed)
    "ext_occ_cap_S_01": lambda: make_space(dict(_OPEN, warp_size=1, float_size=1), "S", 0, 1,
                                           bounds=(256, 256, 512, 512, 64),
                                           min_threads_per_multi_processor=1 << 30, min_fmas_per_load=0,
                                           max_blocks_per_multi_processor=65534, max_registers_per_thread=2),
    # min_fmas 2^20 (every L6 point fails low_fmas)
    "ext_fmas_cap_D_00": lambda: make_space(K40C_DEVICE, "D", 0, 0, bounds=(64, 64, 256, 256, 256),
                                            min_fmas_per_load=1 << 20),
}


def extreme(name: str) -> dict:
    return EXTREME[name]()


def fuzz_space(seed: int, max_bound: int = 24) -> dict:
    """Seeded random small space (SURVEY §8(d) fuzz recipe): bounds in
    [1, max_bound]; warp_size in {4, 8, 16, 32}; max_threads_per_block in
    [warp, 1024]; shared-memory and register limits scaled by a factor in
    [1/64, 1]; thresholds min_threads in [0, 512], min_fmas in [0, 4]; random
    precision and transposes; explicit Fig 9 values."""
    r = random.Random(seed)
    warp = r.choice((4, 8, 16, 32))
    dev = dict(K40C_DEVICE if r.random() < 0.5 else B200_DEVICE)
    dev["warp_size"] = warp
    dev["max_threads_per_block"] = r.randint(warp, 1024)
    f_smem = r.uniform(1.0 / 64, 1.0)
    f_regs = r.uniform(1.0 / 64, 1.0)
    dev["max_shared_mem_per_block"] = max(1, int(dev["max_shared_mem_per_block"] * f_smem))
    dev["max_shmem_per_multi_processor"] = max(1, int(dev["max_shmem_per_multi_processor"] * f_smem))
    dev["max_regs_per_block"] = max(1, int(dev["max_regs_per_block"] * f_regs))
    dev["max_registers_per_multi_processor"] = max(1, int(dev["max_registers_per_multi_processor"] * f_regs))
    dev["float_size"] = r.choice((1, 2, 4, 8))
    fig9 = dict(max_blocks_per_multi_processor=r.choice((1, 2, 4, 8, 16, 32)),
                max_warps_per_multi_processor=r.choice((16, 32, 48, 64)),
                max_registers_per_thread=r.choice((8, 16, 32, 63, 128, 255)))
    bounds = tuple(r.randint(1, max_bound) for _ in range(5))
    return make_space(dev, r.choice(PRECISIONS), r.randint(0, 1), r.randint(0, 1),
                      bounds=bounds,
                      min_threads_per_multi_processor=r.randint(0, 512),
                      min_fmas_per_load=r.randint(0, 4), **fig9)

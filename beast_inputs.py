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

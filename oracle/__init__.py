"""ORACLE — TEST INFRASTRUCTURE ONLY.

Plain CPU implementations of the BEAST GEMM search space (PAPER.md Figs 8-15)
used to prove the CUDA path correct.  Only tests/, __graft_entry__.smoke()
and bench.py's cpu_baseline / `--impl reference` legs may import this package.
It shares no code with paper_conf_ipps_luszczekgkdd16_b200/ and never imports
it.

Modules
  beast_oracle.c  canonical hoisted nest, brute force, per-point predicate
                  evaluator, digest (C, int64) — loaded here through ctypes.
  analytic.py     independent divisor-based counter (pin P5 of DESIGN.md).
  literal.py      line-by-line Python transcription of Figs 11-15 run by a
                  generic dependence-driven evaluator (pin P7).
  closed_form.py  closed-form size of the unpruned space (pin P6).

Parity status: every function here is pinned by tests/test_oracle_*.py; see
DESIGN.md "Oracle pins".
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "beast_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lock = threading.Lock()
_lib = None

FIELDS = (
    "max_threads_per_block", "max_threads_dim_x", "max_threads_dim_y",
    "max_shared_mem_per_block", "warp_size", "max_regs_per_block",
    "max_threads_per_multi_processor", "cuda_major", "cuda_minor",
    "max_registers_per_multi_processor", "max_shmem_per_multi_processor", "float_size",
    "max_blocks_per_multi_processor", "max_warps_per_multi_processor", "max_registers_per_thread",
    "precision_double", "arithmetic_complex", "trans_a", "trans_b",
    "min_threads_per_multi_processor", "min_fmas_per_load",
    "dim_m_max", "dim_n_max", "blk_m_max", "blk_n_max", "blk_k_max",
)

PREDICATES = (
    "over_max_threads", "over_max_regs_per_thread", "over_max_regs_per_block",
    "over_max_shmem", "low_occupancy_regs", "low_occupancy_shmem", "low_fmas",
    "partial_warps", "cant_reshape_a1", "cant_reshape_b1", "cant_reshape_a2",
    "cant_reshape_b2",
)

DERIVED = (
    "threads_per_block", "thr_m", "thr_n", "regs_per_thread", "regs_per_block",
    "shmem_per_block", "max_blocks_by_regs", "max_threads_by_regs",
    "max_blocks_by_shmem", "max_threads_by_shmem", "loads_per_thread",
    "loads_per_block", "fmas_per_thread", "fmas_per_block", "fmas_per_load",
)


class OracleSpace(ctypes.Structure):
    _fields_ = [(f, ctypes.c_int64) for f in FIELDS]


def build(force: bool = False) -> str:
    """Compile beast_oracle.c into liboracle.so (gcc -O2, OpenMP)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + ".tmp.%d" % os.getpid()
        subprocess.check_call(["gcc", "-O2", "-std=c99", "-fopenmp", "-fPIC", "-shared",
                               "-o", tmp, _SRC])
        os.replace(tmp, _LIB)
    return _LIB


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB)
            P = ctypes.POINTER
            u64p = P(ctypes.c_uint64)
            L.oracle_nest.argtypes = [P(OracleSpace), ctypes.c_int, u64p, u64p, u64p,
                                      ctypes.c_uint64, u64p, u64p]
            L.oracle_nest.restype = ctypes.c_int
            L.oracle_brute.argtypes = [P(OracleSpace), ctypes.c_int, u64p, u64p, u64p,
                                       ctypes.c_uint64, u64p]
            L.oracle_brute.restype = ctypes.c_int
            L.oracle_point.argtypes = [P(OracleSpace), P(ctypes.c_int64), P(ctypes.c_int64),
                                       P(ctypes.c_int)]
            L.oracle_point.restype = ctypes.c_int
            L.oracle_digest.argtypes = [u64p, ctypes.c_uint64, ctypes.c_uint64]
            L.oracle_digest.restype = ctypes.c_uint64
            L.oracle_resolve.argtypes = [P(OracleSpace), P(OracleSpace)]
            L.oracle_resolve.restype = ctypes.c_int
            L.oracle_fig9_lookup.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int]
            L.oracle_fig9_lookup.restype = ctypes.c_int64
            _lib = L
    return _lib


def to_struct(space: dict) -> OracleSpace:
    """Translate a beast_inputs description into the oracle's struct (Fig 10:
    S = single/real, D = double/real, C = single/complex, Z = double/complex)."""
    p = space["precision"]
    vals = dict(space)
    vals["precision_double"] = 1 if p in ("D", "Z") else 0
    vals["arithmetic_complex"] = 1 if p in ("C", "Z") else 0
    return OracleSpace(*[int(vals.get(f, 0)) for f in FIELDS])


def resolve(space: dict) -> dict:
    out = OracleSpace()
    if lib().oracle_resolve(ctypes.byref(to_struct(space)), ctypes.byref(out)) != 0:
        raise ValueError("invalid space")
    return {f: getattr(out, f) for f in FIELDS}


def fig9_lookup(major: int, minor: int, which: int) -> int:
    return lib().oracle_fig9_lookup(major, minor, which)


def _u64p(a):
    return a.ctypes.data_as(ctypes.POINTER(ctypes.c_uint64))


def nest(space: dict, threads: int = 1, records: bool = False, digest: bool = True):
    """Run the canonical hoisted nest.  Returns dict(visits[15], rejected[12],
    survivors, digest, records (n x 2 uint64 [hi, lo]) or None)."""
    L = lib()
    s = to_struct(space)
    visits = np.zeros(15, np.uint64)
    rejected = np.zeros(12, np.uint64)
    n = ctypes.c_uint64(0)
    dig = ctypes.c_uint64(0)
    rec = None
    if records:
        # size with a count-only pass first (plain, not fast)
        rc = L.oracle_nest(ctypes.byref(s), threads, _u64p(visits), _u64p(rejected),
                           None, 0, ctypes.byref(n), None)
        if rc != 0:
            raise ValueError("oracle_nest failed: %d" % rc)
        rec = np.zeros((max(int(n.value), 1), 2), np.uint64)
        rc = L.oracle_nest(ctypes.byref(s), threads, _u64p(visits), _u64p(rejected),
                           _u64p(rec), rec.shape[0], ctypes.byref(n), ctypes.byref(dig))
        rec = rec[: int(n.value)]
    else:
        rc = L.oracle_nest(ctypes.byref(s), threads, _u64p(visits), _u64p(rejected),
                           None, 0, ctypes.byref(n), ctypes.byref(dig) if digest else None)
    if rc != 0:
        raise ValueError("oracle_nest failed: %d" % rc)
    return dict(visits=[int(x) for x in visits], rejected=[int(x) for x in rejected],
                survivors=int(n.value), digest=int(dig.value) if (digest or records) else None,
                records=rec)


def brute(space: dict, threads: int = 1, records: bool = True):
    """Brute force (pin P1).  Returns dict(n_space, true_count[12], survivors,
    records)."""
    L = lib()
    s = to_struct(space)
    n_space = ctypes.c_uint64(0)
    true_count = np.zeros(12, np.uint64)
    n = ctypes.c_uint64(0)
    cap = 1 << 20
    rec = np.zeros((cap, 2), np.uint64) if records else None
    rc = L.oracle_brute(ctypes.byref(s), threads, ctypes.byref(n_space), _u64p(true_count),
                        _u64p(rec) if records else None, cap if records else 0, ctypes.byref(n))
    if rc != 0:
        raise ValueError("oracle_brute failed: %d" % rc)
    if records:
        assert n.value <= cap
        rec = rec[: int(n.value)]
    return dict(n_space=int(n_space.value), true_count=[int(x) for x in true_count],
                survivors=int(n.value), records=rec)


def point(space: dict, v) -> tuple[dict, dict]:
    """Derived variables (Fig 12) and the 12 predicates (Figs 13-15) of one
    explicit 15-tuple, in Fig 11 order."""
    L = lib()
    vv = (ctypes.c_int64 * 15)(*[int(x) for x in v])
    der = (ctypes.c_int64 * 15)()
    pred = (ctypes.c_int * 12)()
    if L.oracle_point(ctypes.byref(to_struct(space)), vv, der, pred) != 0:
        raise ValueError("invalid space")
    return dict(zip(DERIVED, list(der))), dict(zip(PREDICATES, [bool(x) for x in pred]))


def digest(records: np.ndarray, base: int = 0) -> int:
    r = np.ascontiguousarray(records, dtype=np.uint64)
    return int(lib().oracle_digest(_u64p(r), r.shape[0], base))


def unpack(hi: int, lo: int) -> tuple:
    """Decode one packed record (SURVEY §8(b) layout) into the 15-tuple."""
    hi, lo = int(hi), int(lo)
    m12 = 0xFFF
    return ((hi >> 52) & m12, (hi >> 40) & m12, (hi >> 28) & m12, (hi >> 16) & m12,
            (hi >> 4) & m12, (hi >> 1) & 7, hi & 1,
            (lo >> 52) & m12, (lo >> 40) & m12, (lo >> 28) & m12, (lo >> 16) & m12,
            (lo >> 3) & 1, (lo >> 2) & 1, (lo >> 1) & 1, lo & 1)

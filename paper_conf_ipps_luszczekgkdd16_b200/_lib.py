"""ctypes binding of include/beast.h — argument marshalling only.

Every step of the enumeration runs in libbeast.so (CUDA, sm_100a).  There is
no CPU fallback: importing this module fails loudly if the shared library is
missing, and every enumerating call fails (BeastError) without a B200.
PyTorch supplies device memory (the caching allocator backs the library's
scratch; record buffers are torch tensors) and streams.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# BEAST_LIB_PATH (development A/B runs only) selects another in-tree build.
LIB_PATH = os.environ.get("BEAST_LIB_PATH") or os.path.join(_HERE, "libbeast.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(
        "libbeast.so not found at %s — build it with `python -c 'import __graft_entry__ as g; g.build()'` "
        "(there is no CPU fallback)" % LIB_PATH)

_L = ctypes.CDLL(LIB_PATH)

BEAST_OK = 0
BEAST_ERR_INVALID_ARGUMENT = -1
BEAST_ERR_UNSUPPORTED = -2
BEAST_ERR_CAPACITY = -3
BEAST_ERR_WORKSPACE = -4
BEAST_ERR_CUDA = -5

PRECISION = {"S": 0, "D": 1, "C": 2, "Z": 3}


class beast_device_limits(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in (
        "max_threads_per_block", "max_threads_dim_x", "max_threads_dim_y",
        "max_shared_mem_per_block", "warp_size", "max_regs_per_block",
        "max_threads_per_multi_processor", "cuda_major", "cuda_minor",
        "max_registers_per_multi_processor", "max_shmem_per_multi_processor", "float_size",
        "max_blocks_per_multi_processor", "max_warps_per_multi_processor",
        "max_registers_per_thread")]


class beast_settings(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in (
        "trans_a", "trans_b", "min_threads_per_multi_processor", "min_fmas_per_load")]


class beast_bounds(ctypes.Structure):
    _fields_ = [(n, ctypes.c_int32) for n in (
        "dim_m_max", "dim_n_max", "blk_m_max", "blk_n_max", "blk_k_max")]


class beast_stats(ctypes.Structure):
    _fields_ = [("visits", ctypes.c_uint64 * 15), ("rejected", ctypes.c_uint64 * 12),
                ("survivors", ctypes.c_uint64), ("prefixes", ctypes.c_uint64),
                ("valid_a", ctypes.c_uint64), ("tuples", ctypes.c_uint64),
                ("formed", ctypes.c_uint64 * 2), ("checked", ctypes.c_uint64 * 2),
                ("l4_digest", ctypes.c_uint64)]


_cpp = ctypes.POINTER(ctypes.c_char_p)


class beast_ir_desc(ctypes.Structure):
    _fields_ = [("n_constants", ctypes.c_int32), ("constant_names", _cpp),
                ("constant_values", ctypes.POINTER(ctypes.c_int64)),
                ("n_iterators", ctypes.c_int32), ("iterator_names", _cpp), ("iterator_start", _cpp),
                ("iterator_stop", _cpp), ("iterator_step", _cpp),
                ("n_derived", ctypes.c_int32), ("derived_names", _cpp), ("derived_exprs", _cpp),
                ("n_constraints", ctypes.c_int32), ("constraint_names", _cpp), ("constraint_exprs", _cpp)]


ALLOC_FN = ctypes.CFUNCTYPE(ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)
FREE_FN = ctypes.CFUNCTYPE(None, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p, ctypes.c_void_p)

_P = ctypes.POINTER
_vp = ctypes.c_void_p
_u64p = _P(ctypes.c_uint64)
_sig = {
    "beast_abi_version": ([], ctypes.c_int),
    "beast_error_string": ([ctypes.c_int], ctypes.c_char_p),
    "beast_last_error": ([_vp], ctypes.c_char_p),
    "beast_limits_k40c": ([_P(beast_device_limits)], ctypes.c_int),
    "beast_limits_from_device": ([ctypes.c_int, _P(beast_device_limits)], ctypes.c_int),
    "beast_limits_resolve": ([_P(beast_device_limits)], ctypes.c_int),
    "beast_space_create": ([_P(beast_device_limits), ctypes.c_int, _P(beast_settings),
                            _P(beast_bounds), _P(_vp)], ctypes.c_int),
    "beast_space_destroy": ([_vp], None),
    "beast_space_set_allocator": ([_vp, ALLOC_FN, FREE_FN, _vp], ctypes.c_int),
    "beast_space_resolved": ([_vp, _P(beast_device_limits), _P(beast_settings),
                              _P(beast_bounds)], ctypes.c_int),
    "beast_count": ([_vp, ctypes.c_int, ctypes.c_int, _vp, _u64p, _P(beast_stats)], ctypes.c_int),
    "beast_enumerate": ([_vp, ctypes.c_int, ctypes.c_int, _vp, _vp, ctypes.c_uint64, _u64p,
                         _P(beast_stats)], ctypes.c_int),
    "beast_enumerate_to_host": ([_vp, ctypes.c_int, ctypes.c_int, _vp, _vp, ctypes.c_uint64,
                                 _u64p, _P(beast_stats)], ctypes.c_int),
    "beast_digest": ([_vp, ctypes.c_uint64, ctypes.c_uint64, _vp, _u64p], ctypes.c_int),
    "beast_enumerate_async": ([_vp, ctypes.c_int, ctypes.c_int, _vp, _vp, ctypes.c_uint64], ctypes.c_int),
    "beast_wait": ([_vp, _vp, _u64p], ctypes.c_int),
    "beast_enumerate_to_host_async": ([_vp, ctypes.c_int, ctypes.c_int, _vp, _vp, ctypes.c_uint64], ctypes.c_int),
    "beast_count_factorized": ([_vp, ctypes.c_int, ctypes.c_int, _vp, _u64p], ctypes.c_int),
    "beast_enumerate_factorized": ([_vp, ctypes.c_int, ctypes.c_int, _vp, _vp, ctypes.c_uint64, _u64p],
                                   ctypes.c_int),
    "beast_enumerate_stage": ([_vp, ctypes.c_int, ctypes.c_int, _vp, _vp, _u64p], ctypes.c_int),
    "beast_write_at": ([_vp, ctypes.c_int, ctypes.c_int, _vp, _vp, ctypes.c_uint64, _vp, _u64p], ctypes.c_int),
    "beast_sweep_count": ([_P(_vp), ctypes.c_int, _vp, _u64p, _P(beast_stats)], ctypes.c_int),
    "beast_ir_create": ([_P(beast_ir_desc), _P(_vp)], ctypes.c_int),
    "beast_ir_destroy": ([_vp], None),
    "beast_ir_last_error": ([_vp], ctypes.c_char_p),
    "beast_ir_source": ([_vp], ctypes.c_char_p),
    "beast_ir_levels": ([_vp, _P(ctypes.c_int32), _P(ctypes.c_int32)], ctypes.c_int),
    "beast_ir_count": ([_vp, _vp, _u64p, _u64p, _u64p], ctypes.c_int),
    "beast_ir_enumerate": ([_vp, _vp, _vp, ctypes.c_uint64, _u64p, _u64p, _u64p], ctypes.c_int),
    "beast_space_set_timing": ([_vp, ctypes.c_int], ctypes.c_int),
    "beast_last_stage_ms": ([_vp, _P(ctypes.c_float)], ctypes.c_int),
    "beast_last_launches": ([_vp, _u64p, _P(ctypes.c_float), _u64p], ctypes.c_int),
    "beast_last_write_ms": ([_vp, ctypes.POINTER(ctypes.c_float)], ctypes.c_int),
    "beast_last_l4_digest": ([_vp, _u64p], ctypes.c_int),
}
for _name, (_args, _res) in _sig.items():
    _f = getattr(_L, _name)
    _f.argtypes = _args
    _f.restype = _res

EXPORTED = tuple(_sig)


def lib():
    return _L

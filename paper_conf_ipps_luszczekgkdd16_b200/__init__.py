"""B200-native BEAST GEMM search-space enumerator (Luszczek et al., IPDPSW 2016).

Python face of include/beast.h.  The functions named beast_* mirror the C ABI
one to one (argument marshalling only); `Space` is a small convenience
wrapper over them.  All enumeration runs in libbeast.so on the GPU.

    import beast_inputs, paper_conf_ipps_luszczekgkdd16_b200 as beast
    sp = beast.Space.from_desc(beast_inputs.headline())
    n = sp.count()                       # 1,207,600
    rec = sp.enumerate()                 # torch.uint64 (n, 2) [lo, hi] on cuda
"""
from __future__ import annotations

import ctypes

from . import _lib
from ._lib import (BEAST_ERR_CAPACITY, BEAST_OK, PRECISION, beast_bounds,  # noqa: F401
                   beast_device_limits, beast_settings, beast_stats)

STAT_PREDICATES = (
    "over_max_threads", "over_max_regs_per_thread", "over_max_regs_per_block",
    "over_max_shmem", "low_occupancy_regs", "low_occupancy_shmem", "low_fmas",
    "partial_warps", "cant_reshape_a1", "cant_reshape_b1", "cant_reshape_a2",
    "cant_reshape_b2",
)


class BeastError(RuntimeError):
    def __init__(self, status, msg=""):
        self.status = status
        super().__init__("%s (%d)%s" % (_lib.lib().beast_error_string(status).decode(), status,
                                        (": " + msg) if msg else ""))


def _check(rc, handle=None):
    if rc != BEAST_OK:
        msg = _lib.lib().beast_last_error(handle).decode() if handle else ""
        raise BeastError(rc, msg)


def _stream_ptr(stream):
    import torch
    if stream is None:
        stream = torch.cuda.current_stream()
    return ctypes.c_void_p(stream.cuda_stream if hasattr(stream, "cuda_stream") else int(stream))


# ----------------------------------------------------------- C-ABI mirrors
def beast_abi_version() -> int:
    return _lib.lib().beast_abi_version()


def beast_limits_k40c() -> beast_device_limits:
    out = beast_device_limits()
    _check(_lib.lib().beast_limits_k40c(ctypes.byref(out)))
    return out


def beast_limits_from_device(device: int = 0) -> beast_device_limits:
    out = beast_device_limits()
    _check(_lib.lib().beast_limits_from_device(device, ctypes.byref(out)))
    return out


def beast_space_create(limits: beast_device_limits, precision, settings=None, bounds=None):
    h = ctypes.c_void_p()
    p = PRECISION[precision] if isinstance(precision, str) else int(precision)
    _check(_lib.lib().beast_space_create(ctypes.byref(limits), p,
                                         ctypes.byref(settings) if settings is not None else None,
                                         ctypes.byref(bounds) if bounds is not None else None,
                                         ctypes.byref(h)))
    return h


def beast_space_destroy(handle) -> None:
    _lib.lib().beast_space_destroy(handle)


def beast_count(handle, rank=0, world=1, stream=None, stats=False):
    n = ctypes.c_uint64(0)
    st = beast_stats() if stats else None
    _check(_lib.lib().beast_count(handle, rank, world, _stream_ptr(stream), ctypes.byref(n),
                                  ctypes.byref(st) if st is not None else None), handle)
    return (int(n.value), stats_dict(st)) if stats else int(n.value)


def beast_enumerate(handle, out, rank=0, world=1, stream=None, stats=False):
    """out: torch.uint64 CUDA tensor of shape (capacity, 2), contiguous.
    Returns the number of records written (and stats)."""
    n = ctypes.c_uint64(0)
    st = beast_stats() if stats else None
    cap = out.shape[0] if out is not None else 0
    ptr = ctypes.c_void_p(out.data_ptr()) if out is not None and cap else None
    rc = _lib.lib().beast_enumerate(handle, rank, world, _stream_ptr(stream), ptr, cap,
                                    ctypes.byref(n), ctypes.byref(st) if st is not None else None)
    if rc == BEAST_ERR_CAPACITY:
        raise BeastError(rc, "need %d records" % n.value)
    _check(rc, handle)
    return (int(n.value), stats_dict(st)) if stats else int(n.value)


def beast_enumerate_to_host(handle, out, rank=0, world=1, stream=None, stats=False):
    """out: pinned CPU torch.uint64 tensor (capacity, 2)."""
    n = ctypes.c_uint64(0)
    st = beast_stats() if stats else None
    cap = out.shape[0] if out is not None else 0
    ptr = ctypes.c_void_p(out.data_ptr()) if out is not None and cap else None
    rc = _lib.lib().beast_enumerate_to_host(handle, rank, world, _stream_ptr(stream), ptr, cap,
                                            ctypes.byref(n), ctypes.byref(st) if st is not None else None)
    if rc == BEAST_ERR_CAPACITY:
        raise BeastError(rc, "need %d records" % n.value)
    _check(rc, handle)
    return (int(n.value), stats_dict(st)) if stats else int(n.value)


def beast_enumerate_async(handle, out, rank=0, world=1, stream=None) -> None:
    """Enqueue a pass captured by an earlier beast_enumerate with the same
    (rank, world, out) and return without waiting (see beast_wait)."""
    cap = out.shape[0] if out is not None else 0
    ptr = ctypes.c_void_p(out.data_ptr()) if out is not None and cap else None
    _check(_lib.lib().beast_enumerate_async(handle, rank, world, _stream_ptr(stream), ptr, cap), handle)


def beast_enumerate_to_host_async(handle, out, rank=0, world=1, stream=None) -> None:
    """Enqueue the pass captured by the handle's last beast_enumerate_to_host
    for (rank, world) plus the copy of its records into `out` (pinned CPU
    torch.uint64 tensor (capacity, 2)); returns at once (see beast_wait)."""
    cap = out.shape[0] if out is not None else 0
    ptr = ctypes.c_void_p(out.data_ptr()) if out is not None and cap else None
    _check(_lib.lib().beast_enumerate_to_host_async(handle, rank, world, _stream_ptr(stream), ptr, cap), handle)


def beast_wait(handle, stream=None) -> int:
    """Wait for the handle's most recent pass; returns its record count."""
    n = ctypes.c_uint64(0)
    rc = _lib.lib().beast_wait(handle, _stream_ptr(stream), ctypes.byref(n))
    if rc == BEAST_ERR_CAPACITY:
        raise BeastError(rc, "need %d records" % n.value)
    _check(rc, handle)
    return int(n.value)


def beast_count_factorized(handle, rank=0, world=1, stream=None) -> int:
    """Survivor count by the factorised (divisor) evaluation — time to
    solution, not a points/s path."""
    n = ctypes.c_uint64(0)
    _check(_lib.lib().beast_count_factorized(handle, rank, world, _stream_ptr(stream), ctypes.byref(n)), handle)
    return int(n.value)


def beast_enumerate_factorized(handle, out, rank=0, world=1, stream=None) -> int:
    n = ctypes.c_uint64(0)
    cap = out.shape[0] if out is not None else 0
    ptr = ctypes.c_void_p(out.data_ptr()) if out is not None and cap else None
    rc = _lib.lib().beast_enumerate_factorized(handle, rank, world, _stream_ptr(stream), ptr, cap, ctypes.byref(n))
    if rc == BEAST_ERR_CAPACITY:
        raise BeastError(rc, "need %d records" % n.value)
    _check(rc, handle)
    return int(n.value)


def beast_digest(records, base=0, stream=None) -> int:
    """Digest of a CUDA uint64 (n, 2) [lo, hi] record tensor."""
    d = ctypes.c_uint64(0)
    n = records.shape[0]
    _check(_lib.lib().beast_digest(ctypes.c_void_p(records.data_ptr()) if n else None, n, base,
                                   _stream_ptr(stream), ctypes.byref(d)))
    return int(d.value)


def beast_enumerate_stage(handle, d_count, rank=0, world=1, stream=None) -> int:
    """NEXT #2, phase 1: stage shard (rank, world); d_count: 1-element
    int64/uint64 CUDA tensor receiving the shard's record count."""
    n = ctypes.c_uint64(0)
    _check(_lib.lib().beast_enumerate_stage(handle, rank, world, _stream_ptr(stream),
                                            ctypes.c_void_p(d_count.data_ptr()), ctypes.byref(n)), handle)
    return int(n.value)


def beast_write_at(handle, out_ptr, capacity, d_counts, rank=0, world=1, stream=None) -> int:
    """NEXT #2, phase 2: write the staged shard at its global offset into the
    device buffer at out_ptr (an int address: a local tensor's data_ptr() or
    rank 0's buffer mapped into this process) of `capacity` records.
    d_counts: CUDA tensor of `world` record counts.  Returns the base offset."""
    base = ctypes.c_uint64(0)
    _check(_lib.lib().beast_write_at(handle, rank, world, _stream_ptr(stream), ctypes.c_void_p(out_ptr), capacity,
                                     ctypes.c_void_p(d_counts.data_ptr()), ctypes.byref(base)), handle)
    return int(base.value)


def beast_sweep_count(handles, stream=None, stats=False):
    """survivor counts (and per-space stats) of a batch
    of spaces, their counting passes run concurrently (include/beast.h)."""
    n = len(handles)
    arr = (ctypes.c_void_p * max(n, 1))(*[h.value if isinstance(h, ctypes.c_void_p) else h for h in handles])
    cnt = (ctypes.c_uint64 * max(n, 1))()
    st = (beast_stats * max(n, 1))() if stats else None
    _check(_lib.lib().beast_sweep_count(arr, n, _stream_ptr(stream), cnt, st))
    counts = [int(cnt[i]) for i in range(n)]
    return (counts, [stats_dict(st[i]) for i in range(n)]) if stats else counts


def sweep(spaces, stream=None, stats=False):
    """beast_sweep_count over Space objects."""
    return beast_sweep_count([sp.handle for sp in spaces], stream=stream, stats=stats)


def stats_dict(st: beast_stats) -> dict:
    return dict(visits=[int(x) for x in st.visits], rejected=[int(x) for x in st.rejected],
                survivors=int(st.survivors), prefixes=int(st.prefixes),
                valid_a=int(st.valid_a), tuples=int(st.tuples),
                formed=[int(x) for x in st.formed], checked=[int(x) for x in st.checked],
                l4_digest=int(st.l4_digest), points=int(sum(st.visits)))


# ----------------------------------------------------------- convenience
def limits_from_desc(desc: dict) -> beast_device_limits:
    return beast_device_limits(*[int(desc.get(f, 0)) for f, _ in beast_device_limits._fields_])


class Space:
    """Owns one beast_space handle; scratch comes from torch's caching
    allocator on the current device."""

    def __init__(self, limits: beast_device_limits, precision, settings=None, bounds=None,
                 torch_alloc: bool = True):
        self.handle = beast_space_create(limits, precision, settings, bounds)
        self._cb = None
        if torch_alloc:
            self._install_torch_allocator()

    @classmethod
    def from_desc(cls, desc: dict, **kw):
        """desc: a beast_inputs space description."""
        s = beast_settings(desc["trans_a"], desc["trans_b"],
                           desc["min_threads_per_multi_processor"], desc["min_fmas_per_load"])
        b = beast_bounds(desc["dim_m_max"], desc["dim_n_max"], desc["blk_m_max"],
                         desc["blk_n_max"], desc["blk_k_max"])
        return cls(limits_from_desc(desc), desc["precision"], s, b, **kw)

    def _install_torch_allocator(self):
        import torch
        dev = torch.cuda.current_device()

        def _alloc(nbytes, stream, ctx):
            try:
                return torch.cuda.caching_allocator_alloc(int(nbytes), dev, stream or 0)
            except Exception:
                return None

        def _free(ptr, nbytes, stream, ctx):
            torch.cuda.caching_allocator_delete(ptr)

        self._cb = (_lib.ALLOC_FN(_alloc), _lib.FREE_FN(_free))
        _check(_lib.lib().beast_space_set_allocator(self.handle, self._cb[0], self._cb[1], None))

    def resolved(self) -> dict:
        lim, st, bd = beast_device_limits(), beast_settings(), beast_bounds()
        _check(_lib.lib().beast_space_resolved(self.handle, ctypes.byref(lim), ctypes.byref(st),
                                               ctypes.byref(bd)))
        d = {f: getattr(lim, f) for f, _ in lim._fields_}
        d.update({f: getattr(st, f) for f, _ in st._fields_})
        d.update({f: getattr(bd, f) for f, _ in bd._fields_})
        return d

    def count(self, rank=0, world=1, stream=None, stats=False):
        return beast_count(self.handle, rank, world, stream, stats)

    def enumerate(self, rank=0, world=1, stream=None, stats=False, out=None):
        """Returns the shard's records as a CUDA uint64 tensor (n, 2) [lo, hi]
        (a view of `out` if given), plus stats if requested."""
        import torch
        if out is None:
            n = self.count(rank, world, stream)
            out = torch.empty((max(n, 1), 2), dtype=torch.uint64, device="cuda")
        r = beast_enumerate(self.handle, out, rank, world, stream, stats)
        n = r[0] if stats else r
        return (out[:n], r[1]) if stats else out[:n]

    def count_factorized(self, rank=0, world=1, stream=None):
        return beast_count_factorized(self.handle, rank, world, stream)

    def enumerate_factorized(self, rank=0, world=1, stream=None, out=None):
        import torch
        if out is None:
            n = self.count_factorized(rank, world, stream)
            out = torch.empty((max(n, 1), 2), dtype=torch.uint64, device="cuda")
        n = beast_enumerate_factorized(self.handle, out, rank, world, stream)
        return out[:n]

    def set_timing(self, enable=True):
        _check(_lib.lib().beast_space_set_timing(self.handle, int(enable)))

    def last_stage_ms(self):
        ms = (ctypes.c_float * 5)()
        _check(_lib.lib().beast_last_stage_ms(self.handle, ms))
        return list(ms)

    def last_launches(self):
        k, ms, n = ctypes.c_uint64(0), ctypes.c_float(0), ctypes.c_uint64(0)
        _check(_lib.lib().beast_last_launches(self.handle, ctypes.byref(k), ctypes.byref(ms),
                                              ctypes.byref(n)))
        return int(k.value), float(ms.value), int(n.value)

    def last_write_ms(self):
        ms = ctypes.c_float(0)
        _check(_lib.lib().beast_last_write_ms(self.handle, ctypes.byref(ms)))
        return float(ms.value)

    def last_l4_digest(self):
        """Digest of the L4 survivor list of the last pass (beast_last_l4_digest)."""
        d = ctypes.c_uint64(0)
        _check(_lib.lib().beast_last_l4_digest(self.handle, ctypes.byref(d)), self.handle)
        return int(d.value)

    def close(self):
        if self.handle:
            beast_space_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


def unpack(lo: int, hi: int) -> tuple:
    """15-tuple of a packed record (include/beast.h layout)."""
    lo, hi = int(lo), int(hi)
    m = 0xFFF
    return ((hi >> 52) & m, (hi >> 40) & m, (hi >> 28) & m, (hi >> 16) & m, (hi >> 4) & m,
            (hi >> 1) & 7, hi & 1, (lo >> 52) & m, (lo >> 40) & m, (lo >> 28) & m,
            (lo >> 16) & m, (lo >> 3) & 1, (lo >> 2) & 1, (lo >> 1) & 1, lo & 1)


# ----------------------------------------------------------- NEXT #4: generic space IR
class IRSpace:
    """A space in the generic IR (include/beast.h beast_ir_desc; the spec dict
    format of oracle/ir.py: constants, iterators [name, start, stop, step],
    derived [name, expr], constraints [name, expr]), compiled by the library
    with NVRTC for sm_100a.  This class only marshals the strings."""

    def __init__(self, spec: dict):
        import torch  # noqa: F401  (CUDA context on the current device)
        enc = lambda xs: (ctypes.c_char_p * max(len(xs), 1))(*[x.encode() for x in xs])  # noqa: E731
        consts = spec.get("constants", {})
        its = spec["iterators"]
        der = spec.get("derived", [])
        con = spec.get("constraints", [])
        self.names = [i[0] for i in its]
        self.constraint_names = [c[0] for c in con]
        self.derived_names = [d[0] for d in der]
        self._keep = [enc(list(consts)), (ctypes.c_int64 * max(len(consts), 1))(*[int(v) for v in consts.values()]),
                      enc([i[0] for i in its]), enc([str(i[1]) for i in its]), enc([str(i[2]) for i in its]),
                      enc([str(i[3]) for i in its]), enc([d[0] for d in der]), enc([d[1] for d in der]),
                      enc([c[0] for c in con]), enc([c[1] for c in con])]
        k = self._keep
        cp = lambda a: ctypes.cast(a, _lib._cpp)  # noqa: E731
        desc = _lib.beast_ir_desc(len(consts), cp(k[0]), ctypes.cast(k[1], ctypes.POINTER(ctypes.c_int64)),
                                  len(its), cp(k[2]), cp(k[3]), cp(k[4]), cp(k[5]),
                                  len(der), cp(k[6]), cp(k[7]), len(con), cp(k[8]), cp(k[9]))
        h = ctypes.c_void_p()
        rc = _lib.lib().beast_ir_create(ctypes.byref(desc), ctypes.byref(h))
        if rc != 0:
            msg = _lib.lib().beast_ir_last_error(h).decode() if h.value else ""
            if h.value:
                _lib.lib().beast_ir_destroy(h)
            raise BeastError(rc, msg)
        self.handle = h

    def _err(self, rc):
        if rc != 0:
            raise BeastError(rc, _lib.lib().beast_ir_last_error(self.handle).decode())

    @property
    def source(self) -> str:
        return _lib.lib().beast_ir_source(self.handle).decode()

    def levels(self) -> dict:
        d = (ctypes.c_int32 * max(len(self.derived_names), 1))()
        c = (ctypes.c_int32 * max(len(self.constraint_names), 1))()
        self._err(_lib.lib().beast_ir_levels(self.handle, d, c))
        out = {n: i for i, n in enumerate(self.names)}
        out.update({n: int(d[i]) for i, n in enumerate(self.derived_names)})
        out.update({n: int(c[i]) for i, n in enumerate(self.constraint_names)})
        return out

    def count(self, stream=None) -> dict:
        n = ctypes.c_uint64(0)
        v = (ctypes.c_uint64 * max(len(self.names), 1))()
        r = (ctypes.c_uint64 * max(len(self.constraint_names), 1))()
        self._err(_lib.lib().beast_ir_count(self.handle, _stream_ptr(stream), ctypes.byref(n), v, r))
        return dict(survivors=int(n.value), visits=[int(x) for x in v[:len(self.names)]],
                    rejected=[int(x) for x in r[:len(self.constraint_names)]])

    def enumerate(self, stream=None):
        """Returns (int64 CUDA tensor [survivors, n_iterators], stats dict)."""
        import torch
        st = self.count(stream)
        out = torch.empty((max(st["survivors"], 1), len(self.names)), dtype=torch.int64, device="cuda")
        n = ctypes.c_uint64(0)
        v = (ctypes.c_uint64 * max(len(self.names), 1))()
        r = (ctypes.c_uint64 * max(len(self.constraint_names), 1))()
        self._err(_lib.lib().beast_ir_enumerate(self.handle, _stream_ptr(stream), ctypes.c_void_p(out.data_ptr()),
                                               out.shape[0], ctypes.byref(n), v, r))
        return out[:int(n.value)], dict(survivors=int(n.value), visits=[int(x) for x in v[:len(self.names)]],
                                         rejected=[int(x) for x in r[:len(self.constraint_names)]])

    def close(self):
        if getattr(self, "handle", None) is not None and self.handle.value:
            _lib.lib().beast_ir_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()


"""ORACLE — TEST INFRASTRUCTURE ONLY.  Reference for SURVEY §8(f) NEXT #4,
the generic space IR: a space written as BEAST-style iterators, derived
variables and constraints (§V-VIII: iterators whose
ranges depend on other iterators, expressions, and "@condition"s where True
prunes, reading A5) enumerated by plain nested loops, exactly as the paper's
generated C does: loops in listing order, every derived
variable computed and every constraint tested as soon as the last iterator it
reads is bound (the level-set rule), constraints of one level in listing
order, the first True one rejecting the point.

An IR spec is data (a dict, also used as the input of the CUDA path, which
shares no code with this file):

    {"constants":   {"N": 16, ...},                     # int64 constants
     "iterators":   [[name, start, stop, step], ...],   # C int64 expressions;
                                                         # values start, start+step, ...
                                                         # while < stop (step > 0) or > stop
     "derived":     [[name, expr], ...],                 # C int64 expressions, listing order
     "constraints": [[name, expr], ...]}                 # C expressions, nonzero prunes

This module writes that spec out as ONE plain C function of nested for
loops (gcc -O1; C semantics for / and %, int64) and runs it.  A variable's
level is the deepest iterator it reads, directly or through derived
variables.  Results: survivors, per-level visits (loop-body executions),
per-constraint first-failing rejections and, optionally, the survivor
tuples in enumeration (= canonical, lexicographic) order.
"""
from __future__ import annotations

import ctypes
import hashlib
import os
import re
import subprocess
import tempfile

import numpy as np

_IDENT = re.compile(r"[A-Za-z_][A-Za-z_0-9]*")


def _reads(expr: str) -> set:
    return set(_IDENT.findall(expr))


def levels(spec: dict) -> dict:
    """Level (0-based iterator index) of every iterator, derived variable and
    constraint; -1 = depends on constants only."""
    lev = {c: -1 for c in spec.get("constants", {})}
    for i, (name, *_r) in enumerate(spec["iterators"]):
        lev[name] = i
    out = {}
    for i, (name, *_r) in enumerate(spec["iterators"]):
        out[name] = i
    for name, expr in spec.get("derived", []):
        lev[name] = max([-1] + [lev[r] for r in _reads(expr) if r in lev])
        out[name] = lev[name]
    for name, expr in spec.get("constraints", []):
        out[name] = max([-1] + [lev[r] for r in _reads(expr) if r in lev])
    return out


def c_source(spec: dict) -> str:
    """The nested-loop C program of the spec (one function, `ir_run`)."""
    its = spec["iterators"]
    der = spec.get("derived", [])
    con = spec.get("constraints", [])
    lev = levels(spec)
    n = len(its)
    L = []
    L.append("typedef long long i64;")
    L.append("int ir_run(i64 *visits, i64 *rejected, i64 *survivors, i64 *rec, i64 cap) {")
    for k, v in spec.get("constants", {}).items():
        L.append("  const i64 %s = (i64)(%dLL);" % (k, int(v)))
    L.append("  i64 nsurv = 0;")
    # constant-level derived variables and constraints
    for name, expr in der:
        if lev[name] < 0:
            L.append("  const i64 %s = (i64)(%s);" % (name, expr))
    pre = [(j, e) for j, (nm, e) in enumerate(con) if lev[nm] < 0]
    depth = 1
    ind = "  "
    if pre:
        L.append(ind + "if (" + " || ".join("(%s)" % e for _, e in pre) + ") {")
        for j, e in pre:
            L.append(ind + "  if (%s) { rejected[%d]++; goto done; }" % (e, j))
        L.append(ind + "}")
    for i, (name, start, stop, step) in enumerate(its):
        ind = "  " * depth
        L.append(ind + "{ const i64 _st%d = (i64)(%s), _hi%d = (i64)(%s), _sp%d = (i64)(%s);" %
                 (i, start, i, stop, i, step))
        L.append(ind + "  if (_sp%d == 0) return -1;" % i)
        L.append(ind + "  for (i64 %s = _st%d; _sp%d > 0 ? %s < _hi%d : %s > _hi%d; %s += _sp%d) {" %
                 (name, i, i, name, i, name, i, name, i))
        L.append(ind + "    visits[%d]++;" % i)
        for dn, de in der:
            if lev[dn] == i:
                L.append(ind + "    const i64 %s = (i64)(%s);" % (dn, de))
        for j, (cn, ce) in enumerate(con):
            if lev[cn] == i:
                L.append(ind + "    if (%s) { rejected[%d]++; continue; }" % (ce, j))
        depth += 2
    ind = "  " * depth
    L.append(ind + "if (rec && nsurv < cap) {")
    for i, (name, *_r) in enumerate(its):
        L.append(ind + "  rec[nsurv * %d + %d] = %s;" % (n, i, name))
    L.append(ind + "}")
    L.append(ind + "nsurv++;")
    for i in reversed(range(n)):
        depth -= 2
        L.append("  " * depth + "  }")
        L.append("  " * depth + "}")
    if pre:
        L.append("done:")
    L.append("  *survivors = nsurv;")
    L.append("  return 0;")
    L.append("}")
    return "\n".join(L) + "\n"


_CACHE = {}


def _compile(src: str):
    key = hashlib.sha1(src.encode()).hexdigest()[:16]
    if key in _CACHE:
        return _CACHE[key]
    d = os.path.join(tempfile.gettempdir(), "beast_ir_oracle")
    os.makedirs(d, exist_ok=True)
    so = os.path.join(d, "ir_%s.so" % key)
    if not os.path.exists(so):
        c = os.path.join(d, "ir_%s.c" % key)
        with open(c, "w") as f:
            f.write(src)
        tmp = so + ".%d" % os.getpid()
        subprocess.check_call(["gcc", "-O1", "-shared", "-fPIC", "-o", tmp, c])
        os.replace(tmp, so)
    lib = ctypes.CDLL(so)
    fn = lib.ir_run
    P = ctypes.POINTER(ctypes.c_int64)
    fn.argtypes = [P, P, P, P, ctypes.c_int64]
    fn.restype = ctypes.c_int
    _CACHE[key] = fn
    return fn


def run(spec: dict, records: bool = False, capacity: int = 1 << 24) -> dict:
    """Enumerate the spec.  Returns dict(survivors, visits[n_iter],
    rejected[n_constraints], records (int64 [survivors, n_iter]) if asked)."""
    fn = _compile(c_source(spec))
    n = len(spec["iterators"])
    visits = np.zeros(n, np.int64)
    rej = np.zeros(max(len(spec.get("constraints", [])), 1), np.int64)
    surv = np.zeros(1, np.int64)
    P = ctypes.POINTER(ctypes.c_int64)
    if records:
        rec = np.zeros((capacity, n), np.int64)
        rc = fn(visits.ctypes.data_as(P), rej.ctypes.data_as(P), surv.ctypes.data_as(P), rec.ctypes.data_as(P),
                capacity)
    else:
        rc = fn(visits.ctypes.data_as(P), rej.ctypes.data_as(P), surv.ctypes.data_as(P), None, 0)
    if rc != 0:
        raise ValueError("iterator with step 0")
    out = dict(survivors=int(surv[0]), visits=[int(x) for x in visits],
               rejected=[int(x) for x in rej[:len(spec.get("constraints", []))]])
    if records:
        if out["survivors"] > capacity:
            raise ValueError("capacity %d < %d survivors" % (capacity, out["survivors"]))
        out["records"] = rec[:out["survivors"]].copy()
    return out

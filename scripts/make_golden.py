"""Write tests/golden/expected.json from the ORACLE ONLY (oracle/ + the input
descriptions of beast_inputs.py).  No value here comes from the CUDA path.

    python scripts/make_golden.py [--threads N] [--only NAME ...]

For every named space: survivors, visits[15], rejected[12], N_canon, the
SURVEY §8(b) digest, the first and last packed records (hex hi/lo), from the
canonical nest (oracle_nest), plus the L7 prefix count and the number of valid
A-read grids from the analytic counter (oracle/analytic.py).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import beast_inputs as bi  # noqa: E402
import oracle  # noqa: E402
import oracle.analytic  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "expected.json")


def spaces():
    out = {}
    for p in bi.PRECISIONS:
        for ta, tb in bi.TRANSPOSES:
            out["tiny_%s_%d%d" % (p, ta, tb)] = bi.tiny(p, ta, tb)
    out["micro_C_00"] = bi.micro("C")
    for p in bi.PRECISIONS:
        for ta, tb in bi.TRANSPOSES:
            out["k40c_%s_%d%d" % (p, ta, tb)] = bi.k40c(p, ta, tb)
    for b in (64, 256, 512):
        out["widened%d_k40c_D_00" % b] = bi.widened(b, "k40c")
        out["widened%d_b200_D_00" % b] = bi.widened(b, "b200")
    out["b200_48k_D_00"] = bi.b200("D", smem_48k=True)
    out["b200_48k_S_00"] = bi.b200("S", smem_48k=True)
    for p in ("D", "Z", "C", "S"):
        for ta, tb in bi.TRANSPOSES:
            out["b200_%s_%d%d" % (p, ta, tb)] = bi.b200(p, ta, tb)
    out["maxbound_k40c_D_00"] = bi.maxbound("k40c", "D")
    out["maxbound_k40c_Z_11"] = bi.maxbound("k40c", "Z", 1, 1)
    out["maxbound_b200_D_00"] = bi.maxbound("b200", "D")
    for name in bi.EXTREME:                 # the admitted-range edge spaces
        out[name] = bi.extreme(name)
    return out


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--threads", type=int, default=os.cpu_count())
    ap.add_argument("--only", nargs="*")
    args = ap.parse_args()
    data = {}
    if os.path.exists(OUT):
        with open(OUT) as f:
            data = json.load(f)
    for name, sp in spaces().items():
        if args.only and name not in args.only:
            continue
        if not args.only and name in data:
            continue
        t = time.time()
        r = oracle.nest(sp, threads=args.threads, records=False, digest=True)
        # first / last records: rerun the nest keeping records only when small
        first = last = None
        if r["survivors"] and r["survivors"] <= 30_000_000:
            rr = oracle.nest(sp, threads=args.threads, records=True)
            assert rr["digest"] == r["digest"]
            first = ["%016x" % rr["records"][0, 0], "%016x" % rr["records"][0, 1]]
            last = ["%016x" % rr["records"][-1, 0], "%016x" % rr["records"][-1, 1]]
            del rr
        a = oracle.analytic.count(sp)
        assert a["visits"] == r["visits"] and a["rejected"] == r["rejected"], name
        data[name] = dict(space=sp, survivors=r["survivors"], visits=r["visits"],
                          rejected=r["rejected"], n_canon=sum(r["visits"]),
                          digest="0x%016x" % r["digest"], first=first, last=last,
                          prefixes=a["prefixes"], valid_a=a["valid_a"])
        print("%-24s survivors %12d  N_canon %16d  digest %s  %.1fs" % (
            name, r["survivors"], sum(r["visits"]), data[name]["digest"], time.time() - t),
            flush=True)
        with open(OUT + ".tmp", "w") as f:
            json.dump(data, f, indent=1, sort_keys=True)
        os.replace(OUT + ".tmp", OUT)


if __name__ == "__main__":
    main()

"""Write tests/golden/wide_fuzz.json from the ORACLE ONLY: the wide fuzz block
(seeds 200-399, beast_inputs.fuzz_space_wide) over the library's whole
admitted input range.

    python scripts/make_wide_fuzz.py [--seeds 200 400] [--budget-s 2.0] [--jobs 8]

For every seed the first attempt (fuzz_space_wide(seed, attempt), attempt =
0, 1, ...) whose canonical nest the oracle finishes single-threaded within
--budget-s is kept -- the spaces the GPU tests can afford to re-run through
the oracle -- with its survivors, visits, rejections, digest and the largest
threads_per_block among its survivors.  No value here comes from the CUDA
path.
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

OUT = os.path.join(ROOT, "tests", "golden", "wide_fuzz.json")


def _nest(desc):
    r = oracle.nest(desc, threads=1, records=True, digest=True)
    rec = r["records"]
    t_max = 0
    if len(rec):
        hi = rec[:, 0].astype("uint64")
        t = (hi >> 52) * ((hi >> 40) & 0xfff)
        t_max = int(t.max())
    return dict(survivors=r["survivors"], visits=r["visits"], rejected=r["rejected"],
                n_canon=sum(r["visits"]), digest="0x%016x" % r["digest"], t_max=t_max)


def one_seed(args):
    """Run each attempt in a child interpreter (killed at the budget)."""
    import subprocess
    seed, budget, max_attempts = args
    for attempt in range(max_attempts):
        desc = bi.fuzz_space_wide(seed, attempt)
        t = time.time()
        try:
            out = subprocess.run([sys.executable, os.path.abspath(__file__), "--one", json.dumps(desc)],
                                 capture_output=True, text=True, timeout=budget + 1.0)
        except subprocess.TimeoutExpired:
            continue
        if out.returncode != 0:
            raise RuntimeError("oracle failed on seed %d attempt %d: %s" % (seed, attempt, out.stderr[-2000:]))
        res = json.loads(out.stdout)
        res.update(seed=seed, attempt=attempt, space=desc, oracle_s=time.time() - t)
        if res["oracle_s"] > budget + 1.0:
            continue
        return res
    return dict(seed=seed, attempt=None)


def main():
    if len(sys.argv) == 3 and sys.argv[1] == "--one":
        print(json.dumps(_nest(json.loads(sys.argv[2]))))
        return
    ap = argparse.ArgumentParser()
    ap.add_argument("--seeds", type=int, nargs=2, default=(200, 400))
    ap.add_argument("--budget-s", type=float, default=2.0)
    ap.add_argument("--max-attempts", type=int, default=200)
    ap.add_argument("--jobs", type=int, default=os.cpu_count())
    args = ap.parse_args()
    oracle.lib()   # build once before forking
    seeds = list(range(*args.seeds))
    from concurrent.futures import ThreadPoolExecutor
    with ThreadPoolExecutor(args.jobs) as pool:   # each attempt runs in its own forked process
        res = list(pool.map(one_seed, [(s, args.budget_s, args.max_attempts) for s in seeds]))
    data = {"generator": "beast_inputs.fuzz_space_wide", "budget_s": args.budget_s,
            "note": "oracle-only (scripts/make_wide_fuzz.py); first attempt per seed whose nest the oracle "
                    "finishes single-threaded within budget_s",
            "spaces": {str(r["seed"]): r for r in res}}
    with open(OUT + ".tmp", "w") as f:
        json.dump(data, f, indent=0, sort_keys=True)
    os.replace(OUT + ".tmp", OUT)
    kept = [r for r in res if r.get("attempt") is not None]
    print("kept %d / %d seeds; with survivors %d; t_max > 1024: %d; > 16384: %d" % (
        len(kept), len(res), sum(1 for r in kept if r["survivors"]),
        sum(1 for r in kept if r["t_max"] > 1024), sum(1 for r in kept if r["t_max"] > 16384)))


if __name__ == "__main__":
    main()

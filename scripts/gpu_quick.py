"""Quick GPU sanity run: a few spaces through the C ABI vs the oracle, with
device timings.  Usage: python scripts/gpu_quick.py [names...]"""
from __future__ import annotations

import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

import beast_inputs as bi  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_luszczekgkdd16_b200 as beast  # noqa: E402


def main():
    names = sys.argv[1:] or ["tiny", "micro", "headline"]
    for name in names:
        desc = bi.named(name)
        t0 = time.time()
        with beast.Space.from_desc(desc) as sp:
            sp.set_timing(True)
            n = sp.count()
            rec, st = sp.enumerate(stats=True)
            torch.cuda.synchronize()
            t1 = time.time()
            for _ in range(3):
                rec = sp.enumerate()
            torch.cuda.synchronize()
            ms = sp.last_stage_ms()
            launches = sp.last_launches()
            got = rec.cpu().numpy()
        print("%s: count %d enumerate %d points %d first call %.2fs stage ms %s launches %s"
              % (name, n, len(got), st["points"], t1 - t0, ["%.3f" % x for x in ms], launches), flush=True)
        if st["points"] < 3e9:
            ref = oracle.nest(desc, threads=os.cpu_count(), records=True)
            want = np.stack([ref["records"][:, 1], ref["records"][:, 0]], 1) if ref["survivors"] else np.zeros((0, 2), np.uint64)
            print("   list equal:", got.shape == want.shape and bool(np.array_equal(got, want)),
                  " visits equal:", st["visits"] == ref["visits"], " rejected equal:", st["rejected"] == ref["rejected"])
            if st["visits"] != ref["visits"]:
                print("   gpu visits", st["visits"]); print("   ref visits", ref["visits"])
            if st["rejected"] != ref["rejected"]:
                print("   gpu rej", st["rejected"]); print("   ref rej", ref["rejected"])


if __name__ == "__main__":
    main()

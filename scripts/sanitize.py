"""One enumeration of a small space through the C ABI, checked against the
oracle, for compute-sanitizer runs (memcheck / racecheck / synccheck).
Usage: compute-sanitizer --tool racecheck python scripts/sanitize.py [space]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402

import beast_inputs as bi  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_luszczekgkdd16_b200 as beast  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "tiny"
desc = bi.named(name) if name in bi.NAMED else bi.fuzz_space(int(name))
with beast.Space.from_desc(desc) as sp:
    rec, st = sp.enumerate(stats=True)
    n = sp.count()
    torch.cuda.synchronize()
    got = rec.cpu().numpy()
ref = oracle.nest(desc, records=True)
want = np.stack([ref["records"][:, 1], ref["records"][:, 0]], 1) if ref["survivors"] else np.zeros((0, 2), np.uint64)
print("%s: %d survivors, list equal %s, visits equal %s" % (name, n, np.array_equal(got, want),
                                                          st["visits"] == ref["visits"]))

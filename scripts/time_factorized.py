"""Time to solution: canonical per-point enumeration vs the factorised
(divisor) path, same space, same output."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import beast_inputs as bi  # noqa: E402
import paper_conf_ipps_luszczekgkdd16_b200 as beast  # noqa: E402


def timeit(fn, reps=20):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


for name in sys.argv[1:] or ["headline", "b200_S"]:
    with beast.Space.from_desc(bi.named(name)) as sp:
        n = sp.count()
        out = torch.empty((n, 2), dtype=torch.uint64, device="cuda")
        t_can = timeit(lambda: beast.beast_enumerate(sp.handle, out))
        d_can = beast.beast_digest(out)
        t_fac = timeit(lambda: beast.beast_enumerate_factorized(sp.handle, out))
        d_fac = beast.beast_digest(out)
        print("%s: canonical %.3f ms, factorised %.3f ms (%.1fx), same list: %s"
              % (name, t_can, t_fac, t_can / t_fac, d_can == d_fac))

"""Time the generic IR engine (NEXT #4) on the GEMM space written in the IR
against the specialised kernels on the same space.  Usage: python scripts/ir_time.py [names]"""
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import torch  # noqa: E402

import beast_inputs as bi  # noqa: E402
import ir_specs  # noqa: E402
import oracle  # noqa: E402
import paper_conf_ipps_luszczekgkdd16_b200 as beast  # noqa: E402

for name in sys.argv[1:] or ["tiny", "widened256_k40c", "headline"]:
    desc = bi.named(name) if name in bi.NAMED else bi.make_space(bi.K40C_DEVICE, "D", bounds=int(name))
    spec = ir_specs.gemm_spec(oracle.resolve(desc), desc["precision"])
    t = time.time()
    with beast.IRSpace(spec) as ir:
        tc = time.time() - t
        st = ir.count()
        torch.cuda.synchronize()
        t = time.time()
        st = ir.count()
        torch.cuda.synchronize()
        ti = time.time() - t
    with beast.Space.from_desc(desc) as sp:
        n, s2 = sp.count(stats=True)
        sp.count()
        torch.cuda.synchronize()
        t = time.time()
        sp.count()
        torch.cuda.synchronize()
        tk = time.time() - t
    pts = sum(st["visits"])
    print("%s: survivors %d (kernels %d) points %d | IR compile %.2fs, IR count %.4fs = %.3e pts/s | "
          "specialised count %.5fs = %.3e pts/s | same stats: %s" %
          (name, st["survivors"], n, pts, tc, ti, pts / ti, tk, pts / tk,
           st["visits"] == s2["visits"] and st["rejected"] == s2["rejected"]), flush=True)

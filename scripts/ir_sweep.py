"""IR engine tuning (development): median CUDA-event time of the IR counting
pass on one space for several values of an engine environment knob (read by
the library on every call).  Usage: python scripts/ir_sweep.py SPACE VAR v1 v2 ..."""
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import torch  # noqa: E402

import beast_inputs as bi  # noqa: E402
import ir_specs  # noqa: E402
import paper_conf_ipps_luszczekgkdd16_b200 as beast  # noqa: E402

name, var, vals = sys.argv[1], sys.argv[2], sys.argv[3:]
desc = bi.named(name)
with beast.Space.from_desc(desc) as sp:
    res = sp.resolved()
    ref = sp.count(stats=True)[1]
spec = ir_specs.gemm_spec(res, desc["precision"])
stream = torch.cuda.current_stream().cuda_stream
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")   # L2 flush between reps, as bench.py
with beast.IRSpace(spec) as ir:
    for v in vals:
        if v == "-":
            os.environ.pop(var, None)
        else:
            os.environ[var] = v
        st = ir.count()
        ok = st["visits"] == ref["visits"] and st["rejected"] == ref["rejected"]
        ms = []
        for _ in range(int(os.environ.get("IR_REPS", "5"))):
            if os.environ.get("IR_FLUSH", "1") == "1":
                flush.zero_()
            if os.environ.get("IR_SYNC", "0") == "1":
                torch.cuda.synchronize()
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record()
            ir.count()
            b.record()
            torch.cuda.synchronize()
            ms.append(a.elapsed_time(b))
        print("%s %s=%s: IR count %.3f ms (min %.3f, all %s) stats equal %s" % (
              name, var, v, statistics.median(ms), min(ms), ["%.2f" % x for x in ms], ok),
              flush=True)

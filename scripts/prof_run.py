"""One warmed-up enumeration inside cudaProfilerStart/Stop, for
`ncu --profile-from-start off`.  Usage: python scripts/prof_run.py [workload] [count]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import beast_inputs as bi  # noqa: E402
import paper_conf_ipps_luszczekgkdd16_b200 as beast  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "headline"
mode = sys.argv[2] if len(sys.argv) > 2 else "enumerate"
sp = beast.Space.from_desc(bi.named(name))
n = sp.count()
out = torch.empty((max(n, 1), 2), dtype=torch.uint64, device="cuda")
for _ in range(2):
    beast.beast_enumerate(sp.handle, out)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStart()
if mode == "count":
    sp.count()
else:
    beast.beast_enumerate(sp.handle, out)
torch.cuda.synchronize()
torch.cuda.cudart().cudaProfilerStop()
print("done", name, n)

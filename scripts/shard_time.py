"""Per-shard device time of one pass, every (rank, world) run on ONE GPU one
after another ("virtual ranks"): the compute part of an N-GPU step is the
slowest shard's pass (the NCCL exchange comes on top).  Prints, per world,
each shard's ms, the max, the balance (mean / max) and the implied strong
speedup over world 1.  Usage: python scripts/shard_time.py [workload] [steps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import beast_inputs as bi  # noqa: E402
import paper_conf_ipps_luszczekgkdd16_b200 as beast  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "headline"
steps = int(sys.argv[2]) if len(sys.argv) > 2 else 50
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
stream = torch.cuda.current_stream()
base = None
with beast.Space.from_desc(bi.named(name)) as sp:
    for world in (1, 2, 4, 8):
        per = []
        for rank in range(world):
            n = sp.count(rank=rank, world=world)
            out = torch.empty((max(n, 1), 2), dtype=torch.uint64, device="cuda")
            for _ in range(3):
                beast.beast_enumerate(sp.handle, out, rank, world, stream)
            ms = []
            for _ in range(steps):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                beast.beast_enumerate_async(sp.handle, out, rank, world, stream)
                e1.record(stream)
                e1.synchronize()
                ms.append(e0.elapsed_time(e1))
            beast.beast_wait(sp.handle, stream)
            ms.sort()
            per.append(ms[len(ms) // 2])
            del out
        mx = max(per)
        base = base or mx
        print("%s world %d: shard ms %s | max %.4f  balance %.2f  speedup %.2f" % (
            name, world, " ".join("%.4f" % x for x in per), mx, sum(per) / len(per) / mx, base / mx), flush=True)

"""Per-shard statistics and device time of one pass at world N (virtual
ranks on one GPU): the data behind the shard work estimate (ScanL4Work).
Usage: python scripts/shard_stats.py [workload] [world] [steps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import beast_inputs as bi  # noqa: E402
import paper_conf_ipps_luszczekgkdd16_b200 as beast  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "b200_S"
world = int(sys.argv[2]) if len(sys.argv) > 2 else 8
steps = int(sys.argv[3]) if len(sys.argv) > 3 else 20
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
stream = torch.cuda.current_stream()
with beast.Space.from_desc(bi.named(name)) as sp:
    rows = []
    for rank in range(world):
        rec, st = sp.enumerate(rank=rank, world=world, stats=True)
        n = rec.shape[0]
        out = torch.empty((max(n, 1), 2), dtype=torch.uint64, device="cuda")
        sp.set_timing(True)
        beast.beast_enumerate(sp.handle, out, rank, world, stream)
        stg = []
        ms = []
        for _ in range(steps):
            flush.zero_()
            beast.beast_enumerate(sp.handle, out, rank, world, stream)
            stg.append(sp.last_stage_ms())
        sp.set_timing(False)
        stg.sort(key=lambda x: x[4])
        s = stg[len(stg) // 2]
        rows.append((rank, s, st))
        print("rank %d  total %.4f  prefix %.4f  A %.4f  B %.4f  tail %.4f | prefixes %d V8 %d V9 %d formedA %d "
              "checkedA %d validA %d V10 %d V11 %d formedB %d checkedB %d tuples %d" % (
            rank, s[4], s[0], s[1], s[2], s[3], st["prefixes"], st["visits"][7], st["visits"][8], st["formed"][0],
            st["checked"][0], st["valid_a"], st["visits"][9], st["visits"][10], st["formed"][1], st["checked"][1],
            st["tuples"]), flush=True)
        del out, rec
    mx = max(r[1][4] for r in rows)
    print("balance mean/max %.3f" % (sum(r[1][4] for r in rows) / len(rows) / mx))

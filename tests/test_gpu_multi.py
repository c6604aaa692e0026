"""Two ranks on two GPUs: the NCCL gather and the fused
NVLink gather (dist.FusedGather, symmetric memory) each deliver the golden
canonical list on rank 0, the ranks' redundantly computed L1-L4 lists agree
(digest all-gather), and `bench.py --gpus 2` (self-launched under
torch.distributed.run) reports n_gpus 2.  Skipped when fewer than two GPUs
are visible (the round's GPU box has one; the virtual-rank tests cover the
shard rule on one GPU)."""
from __future__ import annotations

import json
import os
import socket
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
pytestmark = pytest.mark.gpu


def _need_two():
    import torch
    if not torch.cuda.is_available():
        pytest.fail("CUDA device required for -m gpu tests")
    if torch.cuda.device_count() < 2:
        pytest.skip("needs 2 GPUs (%d visible)" % torch.cuda.device_count())


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    sys.path.insert(0, ROOT)
    torch.cuda.set_device(rank)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", rank))
    try:
        import beast_inputs as bi
        import paper_conf_ipps_luszczekgkdd16_b200 as beast
        from paper_conf_ipps_luszczekgkdd16_b200 import dist as bdist
        g = json.load(open(os.path.join(ROOT, "tests", "golden", "expected.json")))["k40c_D_00"]
        res = {}
        with beast.Space.from_desc(bi.headline()) as sp:
            r = bdist.enumerate_distributed(sp, gather=True, stats=True)
            res["replicas"] = bdist.check_replicas(sp.last_l4_digest(), world)
            if rank == 0:
                res["nccl"] = (int(r["total"]), "0x%016x" % beast.beast_digest(r["gathered"]))
                res["visits"] = r["stats"]["visits"]
            fg = bdist.FusedGather(r["total"])
            for _ in range(2):
                total = fg.run(sp)
            torch.cuda.synchronize()
            if rank == 0:
                res["fused"] = (total, "0x%016x" % beast.beast_digest(fg.buf[:total].view(torch.uint64)))
        q.put((rank, res, g["survivors"], g["digest"], g["visits"]))
    except Exception as e:  # pragma: no cover - reported to the parent
        import traceback
        q.put((rank, {"error": traceback.format_exc()}, None, None, None))
    finally:
        dist.destroy_process_group()


def test_two_ranks_nccl_and_fused_gather_golden():
    _need_two()
    import torch.multiprocessing as mp
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _port()
    ps = [ctx.Process(target=_rank, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = {}
    for _ in ps:
        rank, res, n, dig, visits = q.get(timeout=600)
        out[rank] = (res, n, dig, visits)
    for p in ps:
        p.join(timeout=60)
    for rank, (res, *_rest) in out.items():
        assert "error" not in res, res.get("error")
    res, n, dig, visits = out[0]
    assert res["nccl"] == (n, dig)
    assert res["fused"] == (n, dig)
    assert res["visits"] == visits
    assert len(set(res["replicas"])) == 1


def test_bench_two_gpus_self_launch():
    _need_two()
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "5",
                          "--warmup", "3", "--no-cpu-baseline"], cwd=ROOT, capture_output=True, text=True,
                         timeout=900)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["config"]["parallelism"] == "dp2"
    assert d["config"]["survivors"] == 1_207_600 and d["replicas"]["ranks_agree"]
    assert d["sharded_resident"]["value"] > 0

"""World-size-2 gloo tests of the multi-GPU combine (paper_conf_..._b200/dist.py)
on CPU: shard offsets by all_gather, stats all_reduce, canonical gather to
rank 0.  The per-rank shards are contiguous slices of the oracle's list (the
library's shard rule is tested on the GPU by the virtual-rank test)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import beast_inputs
        import oracle
        from paper_conf_ipps_luszczekgkdd16_b200 import dist as bdist
        ref = oracle.nest(beast_inputs.tiny("C"), records=True)
        full = np.stack([ref["records"][:, 1], ref["records"][:, 0]], 1).astype(np.uint64)
        # uneven contiguous shards, one of them empty when world == 3
        cuts = [0, 1000, len(full)] if world == 2 else [0, 0, 5000, len(full)]
        local = torch.from_numpy(full[cuts[rank]:cuts[rank + 1]].view(np.int64).copy())
        offs = bdist.shard_offsets(local.shape[0], world, local.device)
        assert offs == cuts, (offs, cuts)
        gathered = torch.empty((len(full), 2), dtype=torch.int64) if rank == 0 else None
        total = bdist.gather_records(local, gathered, world)
        assert total == len(full)
        if rank == 0:
            assert np.array_equal(gathered.numpy().view(np.uint64), full)
        # stats: rank r contributes its slice; sums must reconstruct
        st = dict(visits=[rank + 1] * 15, rejected=[10 * (rank + 1)] * 12, survivors=cuts[rank + 1] - cuts[rank],
                  prefixes=rank, valid_a=1, tuples=2)
        tot = bdist.combine_stats(st, world)
        assert tot["survivors"] == len(full)
        assert tot["visits"] == [sum(range(1, world + 1))] * 15
        assert tot["valid_a"] == world and tot["points"] == 15 * sum(range(1, world + 1))
        # SURVEY §8(e) replica check: the L4 digests all-gathered; equal ->
        # passes, one rank different -> every rank raises (no rank hangs)
        st.update(l4_digest=0xFEDCBA9876543210, formed=[5, 6], checked=[1, 2])
        tot = bdist.combine_stats(st, world)
        assert tot["l4_digest"] == 0xFEDCBA9876543210 and tot["formed"] == [5 * world, 6 * world]
        assert bdist.check_replicas(0x1234, world) == [0x1234] * world
        try:
            bdist.check_replicas(0x1234 + (rank == world - 1), world)
            raise AssertionError("mismatch not detected")
        except bdist.ReplicaMismatch:
            pass
        q.put((rank, "ok"))
    except Exception as e:  # pragma: no cover - reported to the parent
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_gloo_combine(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in ps:
        p.start()
    res = dict(q.get(timeout=240) for _ in ps)
    for p in ps:
        p.join(timeout=60)
    assert all(v == "ok" for v in res.values()), res

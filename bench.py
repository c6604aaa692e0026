"""Benchmark: search-space points evaluated / s (and survivors / s) of the BEAST
GEMM space enumeration on N B200s (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload NAME] [--impl reference]

A step is one pass of the whole hot path: resolve,
prefix stage L1-L7, flattener, A grids L8-L9, B grids L10-L11, compaction,
write-out of every surviving record into device memory and, for N > 1, the
combine (all_gather of counts -> offsets, all_reduce of the stats, gather of
the survivors to rank 0 in canonical order).  value = N_canon (points of the
canonical nest, every level) / device time per step,
whole job, max over ranks.  The default workload is BASELINE.json configs[1],
the paper's headline space (DGEMM, no transposes, K40c limits, default
bounds).  Inputs are synthetic space descriptions (beast_inputs.py); there is
no data.  --impl reference times the CPU oracle (oracle/, the only reference
this paper-tier run has) on the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "search-space points evaluated/sec and survivors/sec at 1/2/4/8 B200"
UNIT = "points/s"

WORKLOADS = {
    "headline": "BASELINE configs[1]: full 15-dimension DGEMM space, no transposes, Tesla K40c limits "
                "(PAPER.md Figs 8-11), default bounds 1024, thresholds 256/2",
    "b200_S": "BASELINE configs[3]: SGEMM NN with B200 (sm_100) limits, default bounds",
    "b200_C": "BASELINE configs[3]: CGEMM NN with B200 (sm_100) limits, default bounds",
    "b200_D": "BASELINE configs[3]: DGEMM NN with B200 (sm_100) limits, default bounds",
    "widened256_b200": "BASELINE configs[4]: DGEMM NN, B200 limits, blk_m/blk_n/blk_k <= 256",
    "widened256_k40c": "BASELINE configs[4]: DGEMM NN, K40c limits, blk_m/blk_n/blk_k <= 256",
    "k40c_S": "BASELINE configs[2]: SGEMM NN, K40c limits",
}

# Paper timings of this path (context only):
PAPER_CONTEXT = {"python_s": 66948, "c_s": 264, "cpu": "Xeon E5-2650 v3, 1 core"}

# Measured packed-scan ceiling (profiles/r02_micro/README.md, scripts/micro/scan.cu:
# the best 16-pair block body, 8 IMAD + 8 VIADDMNMX, at 64 warps/SM): points
# per clock per SM.
SCAN_CEILING_POINTS_PER_CLK_SM = 134.75


def config_dict(args, n_canon, survivors):
    """The `config` object of both arms (same keys and values, so the
    driver's same-config check compares like with like)."""
    return {"workload": args.workload, "description": WORKLOADS.get(args.workload, args.workload),
            "n_canon": n_canon, "survivors": survivors, "parallelism": "dp%d" % args.gpus,
            "gather": args.gather if args.gpus > 1 else None}


def _load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "sm_max_mhz": 1965.0}, "fallback"


# ---------------------------------------------------------------- clocks
class ClockSampler:
    """SM clock and throttle reasons sampled through NVML every 10 ms during
    the timed region (falls back to nvidia-smi if NVML is unavailable)."""

    REASONS = {  # NVML clocks-event reason bits
        0x8: "hw_slowdown", 0x40: "hw_thermal_slowdown", 0x20: "sw_thermal_slowdown",
        0x4: "sw_power_cap", 0x80: "hw_power_brake_slowdown",
    }

    def __init__(self, index=0):
        self.index = index
        self.sm, self.sm_max, self.reasons = [], None, set()
        self._stop = threading.Event()
        self._t = None

    def start(self):
        def run():
            try:
                import pynvml
                pynvml.nvmlInit()
                h = pynvml.nvmlDeviceGetHandleByIndex(self.index)
                self.sm_max = pynvml.nvmlDeviceGetMaxClockInfo(h, pynvml.NVML_CLOCK_SM)
                while not self._stop.is_set():
                    self.sm.append(pynvml.nvmlDeviceGetClockInfo(h, pynvml.NVML_CLOCK_SM))
                    r = pynvml.nvmlDeviceGetCurrentClocksEventReasons(h)
                    for bit, name in self.REASONS.items():
                        if r & bit:
                            self.reasons.add(name)
                    self._stop.wait(0.01)
            except Exception:
                while not self._stop.is_set():
                    try:
                        out = subprocess.run(["nvidia-smi", "-i", str(self.index),
                                              "--query-gpu=clocks.sm,clocks.max.sm", "--format=csv,noheader,nounits"],
                                             capture_output=True, text=True, timeout=5).stdout.strip()
                        a, b = [float(x) for x in out.split(",")]
                        self.sm.append(a)
                        self.sm_max = b
                    except Exception:
                        pass
                    self._stop.wait(0.1)
        self._t = threading.Thread(target=run, daemon=True)
        self._t.start()

    def stop(self):
        self._stop.set()
        if self._t:
            self._t.join(timeout=10)

    def summary(self):
        if not self.sm:
            return {"sm_mhz": None, "sm_max_mhz": self.sm_max, "reasons": ["unsampled"]}
        return {"sm_mhz": statistics.median(self.sm), "sm_max_mhz": self.sm_max,
                "reasons": sorted(self.reasons), "samples": len(self.sm)}


# ---------------------------------------------------------------- reference arm
def run_reference(args):
    """CPU oracle (oracle/beast_oracle.c, OpenMP over dim_m) on the same
    workload; each step enumerates the whole space (bounded: seconds)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return 0
    import beast_inputs
    import oracle
    desc = beast_inputs.named(args.workload)
    cores = os.cpu_count() or 1
    # Bounded sample: if the whole space per step would make the run longer
    # than ~150 s on this host, each step enumerates the canonical prefix
    # dim_m <= D of the same space (the first L1 values, all inner loops).
    t = time.perf_counter()
    r = oracle.nest(desc, threads=cores, digest=False)
    full_t = time.perf_counter() - t
    sample = "whole %s space per step" % args.workload
    if full_t * (args.steps + args.warmup) > 150.0:
        dmx = oracle.resolve(desc)["dim_m_max"]
        frac = 150.0 / (full_t * (args.steps + args.warmup))
        d = max(1, int(dmx * frac))
        desc = dict(desc, dim_m_max=d)
        sample = "canonical prefix dim_m <= %d of the %s space per step" % (d, args.workload)
    n_canon = None
    survivors = None
    for _ in range(args.warmup - 1):
        r = oracle.nest(desc, threads=cores, digest=False)
    times = []
    for _ in range(args.steps):
        t = time.perf_counter()
        r = oracle.nest(desc, threads=cores, digest=False)
        times.append(time.perf_counter() - t)
        n_canon, survivors = sum(r["visits"]), r["survivors"]
    ms = 1e3 * sum(times) / len(times)
    value = n_canon / (ms / 1e3)
    # the whole workload's size for the config object (the sample may be a prefix)
    if "prefix" in sample:
        import oracle.analytic
        full = oracle.analytic.count(beast_inputs.named(args.workload))
        cfg_canon, cfg_surv = sum(full["visits"]), full["survivors"]
    else:
        cfg_canon, cfg_surv = n_canon, survivors
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": args.gpus,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
        "config": config_dict(args, cfg_canon, cfg_surv),
        "survivors_per_s": survivors / (ms / 1e3),
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "cpu": _cpu_model(),
                         "sample": "%s (%d points), canonical nest, OpenMP over dim_m" % (sample, n_canon)},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)
    return 0


# ---------------------------------------------------------------- GPU arm
def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--workload", default="headline", choices=sorted(WORKLOADS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-sweep", action="store_true", help="skip the batched-sweep (NEXT #3) measurement")
    ap.add_argument("--no-ir", action="store_true", help="skip the generic-IR (NEXT #4) measurement")
    ap.add_argument("--gather", default="nccl", choices=["nccl", "fused"],
                    help="N > 1 survivor gather: NCCL point-to-point (default) or the fused NVLink write-out (NEXT #2)")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        return run_reference(args)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        return relaunch(args)

    import torch
    import torch.distributed as dist

    import beast_inputs
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_ipps_luszczekgkdd16_b200 as beast
    from paper_conf_ipps_luszczekgkdd16_b200 import dist as bdist

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        print("bench.py: --gpus %d but WORLD_SIZE=%d ranks were launched" % (args.gpus, world), file=sys.stderr)
        return 2
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        assert dist.get_world_size() == args.gpus
    desc = beast_inputs.named(args.workload)
    sp = beast.Space.from_desc(desc)
    stream = torch.cuda.current_stream()

    # sizes (and the canonical point count) from one instrumented pass; the
    # ranks' redundantly computed L1-L4 lists are checked equal by digest
    # (combine_stats all-gathers l4_digest)
    _, st_local = sp.enumerate(rank=rank, world=world, stats=True)
    stats = bdist.combine_stats(st_local, world)
    n_canon = stats["points"]
    survivors = stats["survivors"]
    replicas = bdist.check_replicas(sp.last_l4_digest(), world)

    out = torch.empty((max(st_local["survivors"], 1), 2), dtype=torch.uint64, device="cuda")
    gathered = torch.empty((max(survivors, 1), 2), dtype=torch.uint64, device="cuda") if rank == 0 else None
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")   # > 126 MB L2

    fused = bdist.FusedGather(survivors, group=None) if (world > 1 and args.gather == "fused") else None

    def step():
        if fused is not None:
            return fused.run(sp, stream)
        n = beast.beast_enumerate(sp.handle, out, rank, world, stream)
        if world > 1:
            bdist.gather_records(out[:n], gathered, world)
        return n

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    # Timed region: K steps, each = one pass of the whole pipeline enqueued
    # with beast_enumerate_async (the graph the synchronous warm-up calls
    # captured), bracketed by CUDA events on the stream; the L2 flush between
    # steps is outside the events.  No host wait inside a step; every pass's
    # completion and count are checked after the loop (beast_wait: the
    # handle's passes are stream-ordered, so the last one completing implies
    # all did).  Multi-GPU steps add the NCCL gather and stay synchronous.
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    launches = 0
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.3)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    for i in range(args.steps):
        flush.zero_()                     # L2 flush between timed steps (not timed)
        ev[i][0].record(stream)
        if world > 1:
            step()
        else:
            beast.beast_enumerate_async(sp.handle, out, rank, world, stream)
        ev[i][1].record(stream)
        launches += sp.last_launches()[0]
    if world == 1:
        assert beast.beast_wait(sp.handle, stream) == st_local["survivors"]
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks.stop()
    total_ms = sum(a.elapsed_time(b) for a, b in ev)
    if world > 1:
        t = torch.tensor([total_ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        total_ms = float(t.item())
    ms = total_ms / args.steps

    # Sharded-resident: the same passes without the gather --
    # every rank's shard stays in its own HBM (the global list is the
    # concatenation in rank order); device time per step, max over ranks.
    sharded = None
    if world > 1:
        rev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
               for _ in range(args.steps)]
        dist.barrier()
        torch.cuda.synchronize()
        for i in range(args.steps):
            flush.zero_()
            rev[i][0].record(stream)
            beast.beast_enumerate_async(sp.handle, out, rank, world, stream)
            rev[i][1].record(stream)
        assert beast.beast_wait(sp.handle, stream) == st_local["survivors"]
        torch.cuda.synchronize()
        t = torch.tensor([sum(a.elapsed_time(b) for a, b in rev) / args.steps], dtype=torch.float64,
                         device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        sms = float(t.item())
        sharded = {"ms_per_step": sms, "value": n_canon / (sms / 1e3),
                   "how": "beast_enumerate_async per rank, no gather (list resident as N shards); "
                          "CUDA events, max over ranks"}

    # count (beast_count: the same pass without compaction order and
    # write-out), timed on its own: CUDA events around each synchronous call
    cnt_ms = []
    sp.count(rank=rank, world=world, stream=stream)
    for _ in range(max(3, args.steps // 2)):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(stream)
        sp.count(rank=rank, world=world, stream=stream)
        b.record(stream)
        b.synchronize()
        cnt_ms.append(a.elapsed_time(b))
    c_ms = statistics.median(cnt_ms)
    if world > 1:
        t = torch.tensor([c_ms], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        c_ms = float(t.item())
    count_line = {"ms_per_step": c_ms, "value": n_canon / (c_ms / 1e3), "unit": UNIT,
                  "how": "beast_count (survivor count only: no canonical placement, no write-out), "
                         "median of synchronous flushed calls, CUDA events"}

    # Roofline: the dominant kernel's launches timed by the library's CUDA
    # events on the launching stream, over K synchronous flushed steps.
    sp.set_timing(True)
    step()
    a_eval_ms, write_ms = [], []
    for i in range(args.steps):
        flush.zero_()
        step()
        a_eval_ms.append(sp.last_launches()[1])
        write_ms.append(sp.last_write_ms())
    stages = sp.last_stage_ms()
    sp.set_timing(False)

    # e2e: the same metric through the public host-buffer call (list copied
    # back to pinned host memory every step)
    host = torch.empty((max(st_local["survivors"], 1), 2), dtype=torch.uint64).pin_memory()
    for _ in range(2):
        beast.beast_enumerate_to_host(sp.handle, host, rank, world, stream)
    torch.cuda.synchronize()
    e2e_ms = []
    for _ in range(max(3, args.steps // 2)):
        flush.zero_()
        torch.cuda.synchronize()
        t = time.perf_counter()
        beast.beast_enumerate_to_host(sp.handle, host, rank, world, stream)
        e2e_ms.append(1e3 * (time.perf_counter() - t))
    e2e_sync_step = statistics.median(e2e_ms)

    # e2e, pipelined (the headline e2e): three handles of the same space on
    # three streams, beast_enumerate_to_host_async rotating over them, so the
    # copy engine moves one step's list to pinned host memory while the SMs
    # compute the next.  Every step still runs its whole pass, flushes L2
    # first (on its stream) and copies its whole list to the host; the timed
    # region is host wall clock from the first enqueue to the last wait.
    NPIPE = 3
    extra = [beast.Space.from_desc(desc) for _ in range(NPIPE - 1)]
    pipe_sp = [sp] + extra
    pipe_st = [torch.cuda.Stream() for _ in range(NPIPE)]
    pipe_host = [host] + [torch.empty_like(host).pin_memory() for _ in range(NPIPE - 1)]
    pipe_flush = [flush] + [torch.empty_like(flush) for _ in range(NPIPE - 1)]
    for k in range(NPIPE):
        for _ in range(2):
            beast.beast_enumerate_to_host(pipe_sp[k].handle, pipe_host[k], rank, world, pipe_st[k])
    torch.cuda.synchronize()
    n_pipe = max(8, args.steps)
    t = time.perf_counter()
    for i in range(n_pipe):
        k = i % NPIPE
        if i >= NPIPE:
            beast.beast_wait(pipe_sp[k].handle, pipe_st[k])
        with torch.cuda.stream(pipe_st[k]):
            pipe_flush[k].zero_()
        beast.beast_enumerate_to_host_async(pipe_sp[k].handle, pipe_host[k], rank, world, pipe_st[k])
    for k in range(NPIPE):
        got = beast.beast_wait(pipe_sp[k].handle, pipe_st[k])
        assert got == st_local["survivors"], (got, st_local["survivors"])
    e2e_step = 1e3 * (time.perf_counter() - t) / n_pipe
    # Informational (not the reported value): device-only passes of the same
    # handles overlapped on their streams (each still preceded by its own L2
    # flush): how much of one pass's latency-bound phases another pass's
    # compute fills.  The reported value stays the one-pass-at-a-time rate.
    overlapped = None
    if world == 1:
        pipe_out = [out] + [torch.empty_like(out) for _ in range(NPIPE - 1)]
        for k in range(NPIPE):
            beast.beast_enumerate(pipe_sp[k].handle, pipe_out[k], rank, world, pipe_st[k])
        torch.cuda.synchronize()
        t = time.perf_counter()
        for i in range(n_pipe):
            k = i % NPIPE
            if i >= NPIPE:
                beast.beast_wait(pipe_sp[k].handle, pipe_st[k])
            with torch.cuda.stream(pipe_st[k]):
                pipe_flush[k].zero_()
            beast.beast_enumerate_async(pipe_sp[k].handle, pipe_out[k], rank, world, pipe_st[k])
        for k in range(NPIPE):
            assert beast.beast_wait(pipe_sp[k].handle, pipe_st[k]) == st_local["survivors"]
        ov_ms = 1e3 * (time.perf_counter() - t) / n_pipe
        overlapped = {"handles": NPIPE, "ms_per_step": ov_ms, "value": n_canon / (ov_ms / 1e3),
                      "note": "informational: %d passes of the space in flight on %d streams (each with its "
                              "own L2 flush), host wall clock; the reported value is one pass at a time"
                              % (NPIPE, NPIPE)}
        del pipe_out
    for x in extra:
        x.close()
    # the bound of the pipelined e2e: one plain device -> pinned host copy of
    # a list of the same size (copy engine, CUDA events)
    dev_list = torch.empty_like(host, device="cuda")
    copy_ms = []
    for _ in range(10):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        host.copy_(dev_list, non_blocking=True)
        e1.record()
        e1.synchronize()
        copy_ms.append(e0.elapsed_time(e1))
    d2h_copy_ms = statistics.median(copy_ms)
    del dev_list
    del pipe_flush
    if world > 1:
        t = torch.tensor([e2e_step, e2e_sync_step], dtype=torch.float64, device="cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        e2e_step, e2e_sync_step = (float(x) for x in t.tolist())

    # time to solution of the factorised path (the same
    # canonical list, checked by digest); never reported as points/s
    fact = None
    if world == 1:
        n = beast.beast_enumerate(sp.handle, out, stream=stream)
        d_can = beast.beast_digest(out[:n], stream=stream)
        beast.beast_enumerate_factorized(sp.handle, out, stream=stream)
        same = beast.beast_digest(out[:n], stream=stream) == d_can
        n_f = max(3, args.steps // 2)
        fev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(n_f)]
        for i in range(n_f):
            flush.zero_()
            fev[i][0].record(stream)
            beast.beast_enumerate_factorized(sp.handle, out, stream=stream)
            fev[i][1].record(stream)
        torch.cuda.synchronize()
        f_ms = sum(a.elapsed_time(b) for a, b in fev) / n_f
        fact = {"ms_per_step": f_ms, "speedup_vs_canonical": ms / f_ms, "same_list": same,
                "note": "time to solution of the same survivor list by divisor factorisation "
                        "(beast_enumerate_factorized); not a points/s figure"}

    sweep = None
    if world == 1 and not args.no_sweep:
        sweep = sweep_measure(beast, beast_inputs, stream, flush)
    generic_ir = None
    if world == 1 and not args.no_ir:
        generic_ir = ir_measure(beast, desc, stream, flush, ms)

    line = None
    if rank == 0:
        peaks, peak_src = _load_peaks()
        a_ms = statistics.mean(a_eval_ms)
        # survivor write-out (SURVEY §8(d) iii): 16 B per record written by
        # k_place_write, against the HBM copy bandwidth of MEASURED_PEAKS.json
        w_ms = statistics.mean(write_ms) if write_ms and min(write_ms) > 0 else None
        w_bytes = 16 * st_local["survivors"]
        write_out = None
        if w_ms:
            w_gbs = w_bytes / (w_ms * 1e6)
            write_out = {"kernel": "k_place_write (canonical placement fused with the write-out: the 16 records "
                                   "of each tuple as one 256-byte piece at its slot)",
                         "bytes_per_launch": w_bytes, "avg_launch_ms": w_ms,
                         "achieved_GBps": w_gbs, "peak_GBps": peaks["hbm_gbs"], "frac": w_gbs / peaks["hbm_gbs"],
                         "peak_source": "MEASURED_PEAKS.json hbm_gbs (%s; a read+write copy rate, the "
                                        "write-only kernel is compared against it)" % peak_src}
        a_points = st_local["visits"][8]       # this rank's L9 points: its launch evaluates all of them
        # Roofline: every point needs one product and one
        # compare = 2 integer ops.  Peak = issue-bound integer lane rate with
        # 16-bit SIMD (one 32-bit lane instruction carries two 16-bit ops):
        # SMs x 4 sub-partitions x 32 lanes x 2 halves x sm_max_mhz.
        ops_per_point = 2
        sm_count = torch.cuda.get_device_properties(0).multi_processor_count
        lanes = 128                            # integer lane-instructions / clk / SM (4 x 32, ALU + FMA pipes)
        peak_ops = sm_count * lanes * 2 * float(peaks.get("sm_max_mhz", 1965.0)) * 1e6
        achieved = ops_per_point * a_points / (a_ms / 1e3) if a_ms > 0 else 0.0
        scan_ceiling_ops = sm_count * SCAN_CEILING_POINTS_PER_CLK_SM * ops_per_point * \
            float(peaks.get("sm_max_mhz", 1965.0)) * 1e6
        traffic = None
        prof = os.path.join(ROOT, "profiles", "k_eval_traffic.json")
        if os.path.exists(prof):
            try:
                traffic = json.load(open(prof)).get(args.workload)
            except Exception:
                traffic = None
        clk = clocks.summary()
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            cpu = cpu_baseline(desc, n_canon, args.workload)
        line = {
            "metric": METRIC, "value": n_canon / (ms / 1e3), "unit": UNIT, "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": config_dict(args, n_canon, survivors),
            "l2": "flushed between timed steps (256 MiB write, outside the timed events)",
            "survivors_per_s": survivors / (ms / 1e3),
            "gathered": {"ms_per_step": ms, "value": n_canon / (ms / 1e3)} if world > 1 else None,
            "sharded_resident": sharded,
            "count": count_line,
            "replicas": {"l4_digests": ["0x%016x" % d for d in replicas], "ranks_agree": len(set(replicas)) == 1,
                         "how": "digest of each rank's redundantly computed L1-L4 list, all-gathered"},
            "roofline": {"bound": "alu",
                         "kernel": "k_tile_eval<A> (L8-L9 A-read grids; each 512-prefix tile is bucketed by row "
                                   "length in shared memory by the same kernel, so its time includes the "
                                   "flattening that round 1 ran as two separate kernels)",
                         "achieved": achieved / 1e12, "peak": peak_ops / 1e12, "unit": "T int16-ops/s",
                         "frac": achieved / peak_ops if peak_ops else None, "traffic": traffic,
                         "peak_measured_scan": scan_ceiling_ops / 1e12,
                         "frac_measured_scan": achieved / scan_ceiling_ops,
                         "peak_measured_scan_source": "profiles/r02_micro: best packed-scan body %.2f points/clk/SM "
                                                      "(scripts/micro/scan.cu) x SMs x sm_max_mhz x 2 ops"
                                                      % SCAN_CEILING_POINTS_PER_CLK_SM,
                         "algorithmic_ops_per_launch": ops_per_point * a_points,
                         "avg_launch_ms": a_ms,
                         "peak_source": "%d SMs x %d int lane-instr/clk x 2 (16-bit halves) x sm_max_mhz (%s "
                                        "MEASURED_PEAKS.json); 2 int ops per point" % (sm_count, lanes, peak_src),
                         "points_per_s_kernel": a_points / (a_ms / 1e3) if a_ms > 0 else None,
                         "frac_whole_pass": (n_canon / (ms / 1e3)) / (peak_ops / ops_per_point)
                         if peak_ops else None,
                         "frac_whole_pass_how": "canonical points per second of the whole step (all 15 levels, "
                                                "every kernel) against the same peak, one point = 2 ops"},
            "e2e": {"value": n_canon / (e2e_step / 1e3), "unit": UNIT,
                    "h2d_bytes_per_step": 0,
                    "inputs": "a 96-byte space description, resolved into kernel parameters when the handle "
                              "captures its pass; a replayed pass reads no host input",
                    "d2h_bytes_per_step": 16 * st_local["survivors"] + 512,
                    "ms_per_step": e2e_step,
                    "d2h_copy_ms": d2h_copy_ms,
                    "d2h_GBps": host.numel() * 8 / (d2h_copy_ms * 1e6) if d2h_copy_ms > 0 else None,
                    "how": "beast_enumerate_to_host_async on three handles of the space, rotating streams: "
                           "each step = L2 flush + whole pass + copy of its whole list to pinned host memory; "
                           "one step's copy overlaps the next step's pass; host wall clock over %d steps" % n_pipe,
                    "unpipelined": {"value": n_canon / (e2e_sync_step / 1e3), "ms_per_step": e2e_sync_step,
                                    "how": "beast_enumerate_to_host (synchronous), median step"}},
            "write_out": write_out,
            "overlapped_passes": overlapped,
            "gpu_launches": launches,
            "clocks": clk,
            "cpu_baseline": cpu,
            "stages_ms": stages,
            "timing": "value: per-step CUDA events around beast_enumerate_async passes (device time, L2 "
                      "flushed before each step, counts checked after the loop); roofline: k_tile_eval<A> "
                      "launches timed by CUDA events in a second loop of synchronous flushed steps",
            "factorised": fact,
            "sweep": sweep,
            "generic_ir": generic_ir,
            "paper_context": PAPER_CONTEXT,
        }
        print(json.dumps(line), flush=True)
    sp.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()
    return 0


def sweep_measure(beast, beast_inputs, stream, flush, reps=3):
    """the 32 configurations the paper tunes one at a
    time (4 precisions x 4 transposes x {K40c, B200}) counted by one
    beast_sweep_count call (passes concurrent on internal streams) against
    the same 32 counting passes issued one after another; CUDA events on the
    caller's stream, L2 flushed before each repetition."""
    import torch
    descs = [(dev, p, ta, tb) for dev in ("k40c", "b200") for p in beast_inputs.PRECISIONS
             for ta, tb in beast_inputs.TRANSPOSES]
    spaces = [beast.Space.from_desc(getattr(beast_inputs, dev)(p, ta, tb)) for dev, p, ta, tb in descs]
    try:
        counts, stats = beast.sweep(spaces, stream=stream, stats=True)
        points = sum(st["points"] for st in stats)
        beast.sweep(spaces, stream=stream)
        for sp in spaces:
            sp.count(stream=stream)

        def timed(fn):
            ms = []
            for _ in range(reps):
                flush.zero_()
                a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                a.record(stream)
                fn()
                b.record(stream)
                torch.cuda.synchronize()
                ms.append(a.elapsed_time(b))
            return statistics.median(ms)

        got = []
        sweep_ms = timed(lambda: got.append(beast.sweep(spaces, stream=stream)))
        seq_ms = timed(lambda: [sp.count(stream=stream) for sp in spaces])
        assert all(g == counts for g in got)
        # the part overlap cannot hide: every pass's grid-evaluation stages
        # (flattener + A grids, B grids: issue-bound, they fill the GPU),
        # measured one pass at a time with the library's stage events
        eval_ms = 0.0
        for sp in spaces:
            sp.set_timing(True)
            flush.zero_()
            sp.count(stream=stream)
            st_ms = sp.last_stage_ms()
            eval_ms += st_ms[1] + st_ms[2]
            sp.set_timing(False)
        return {"spaces": len(spaces), "configs": "4 precisions x 4 transposes x {K40c, B200}",
                "survivors": sum(counts), "points": points, "ms": sweep_ms, "sequential_ms": seq_ms,
                "points_per_s": points / (sweep_ms / 1e3), "speedup_vs_sequential": seq_ms / sweep_ms,
                "grid_eval_ms": eval_ms,
                "overlap_bound_speedup": seq_ms / max(eval_ms, 1e-9),
                "note": "beast_sweep_count (canonical counting passes, concurrent, largest first over 8 "
                        "streams); each pass evaluates every canonical point of its space.  grid_eval_ms = "
                        "the passes' grid-evaluation stages one at a time (issue-bound, they fill the GPU): "
                        "overlap can hide at most sequential_ms - grid_eval_ms"}
    finally:
        for sp in spaces:
            sp.close()


def ir_measure(beast, desc, stream, flush, canonical_ms, reps=7):
    """the same workload written in the generic space IR
    (tests/ir_specs.gemm_spec: Figs 11-15 as iterators, derived variables and
    constraints), compiled by the library with NVRTC and counted by the
    level-wise IR engine; CUDA events on the caller's stream.  The IR spec's
    constants come from the library's own resolution of the space
    (beast_space_resolved), not from the oracle."""
    import torch
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    import ir_specs
    # the IR engine's level buffers come from the device's stream-ordered
    # pool: hand back what torch's caching allocator holds from the earlier
    # measurements first (otherwise the pool re-maps on every call)
    torch.cuda.synchronize()
    torch.cuda.empty_cache()
    with beast.Space.from_desc(desc) as sp:
        res = sp.resolved()
    spec = ir_specs.gemm_spec(res, desc["precision"])
    t = time.perf_counter()
    try:
        ir = beast.IRSpace(spec)
    except Exception as e:          # no NVRTC on this box: report, do not fail the bench
        return {"error": str(e)[:200]}
    compile_s = time.perf_counter() - t
    with ir:
        try:
            for _ in range(2):
                st = ir.count(stream=stream)
        except Exception as e:
            return {"error": str(e)[:200]}
        ms = []
        for _ in range(reps):
            flush.zero_()
            torch.cuda.synchronize()   # the engine is host-driven (a sync per level): start it on an idle GPU
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(stream)
            ir.count(stream=stream)
            b.record(stream)
            torch.cuda.synchronize()
            ms.append(a.elapsed_time(b))
    m = statistics.median(ms)
    pts = sum(st["visits"])
    return {"ms": m, "ms_min": min(ms), "reps": reps, "points": pts, "points_per_s": pts / (m / 1e3),
            "survivors": st["survivors"],
            "compile_s": compile_s, "vs_specialised": m / canonical_ms,
            "note": "generic IR engine (NVRTC-compiled, level-wise) on the same space; counting pass"}


def _cpu_model():
    """lscpu's model fields plus the microarchitecture they name (Intel
    family 6 model numbers)."""
    info = {}
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for line in out.splitlines():
            k, _, v = line.partition(":")
            info[k.strip()] = v.strip()
    except Exception:
        pass
    if not info:
        try:
            for line in open("/proc/cpuinfo"):
                k, _, v = line.partition(":")
                k = {"model name": "Model name", "cpu family": "CPU family", "model": "Model",
                     "stepping": "Stepping"}.get(k.strip())
                if k and k not in info:
                    info[k] = v.strip()
        except OSError:
            pass
    uarch = {("6", "143"): "Sapphire Rapids", ("6", "207"): "Emerald Rapids", ("6", "173"): "Granite Rapids",
             ("6", "106"): "Ice Lake-SP", ("6", "85"): "Skylake/Cascade Lake-SP"}.get(
        (info.get("CPU family"), info.get("Model")))
    return {"model_name": info.get("Model name"), "family": info.get("CPU family"), "model": info.get("Model"),
            "stepping": info.get("Stepping"), "microarchitecture": uarch,
            "sockets": info.get("Socket(s)"), "cores_per_socket": info.get("Core(s) per socket"),
            "threads_per_core": info.get("Thread(s) per core")}


def _oracle_run(desc, threads, budget_s):
    """Oracle nest on `desc` with `threads` OpenMP threads: the whole space if
    it takes at most budget_s, else the canonical prefix dim_m <= D with D
    doubled from 1 while a run stays under budget_s (the work is far from
    uniform in dim_m, so D is found by measurement).  Returns (D or None for
    the whole space, points, survivors, seconds)."""
    import oracle
    dmx = oracle.resolve(desc)["dim_m_max"]
    d, best = 1, None
    if threads > 1:
        d = dmx                      # OpenMP is over dim_m: a prefix would starve the cores
    while True:
        dd = min(d, dmx)
        t = time.perf_counter()
        r = oracle.nest(desc if dd >= dmx else dict(desc, dim_m_max=dd), threads=threads, digest=False)
        dt = time.perf_counter() - t
        best = (None if dd >= dmx else dd, sum(r["visits"]), r["survivors"], dt)
        if dd >= dmx or dt * 2.5 > budget_s:   # the next doubling would overrun the budget
            return best
        d *= 2


def cpu_baseline(desc, n_canon=None, workload="headline", budget_s=10.0):
    """The oracle nest on this host (SURVEY §8(d) "oracle timing beside it"):
    the bench workload on all cores (the reported value; whole space) and on
    one thread (bounded prefix), plus both rates over BASELINE configs[0..2]
    (tiny DGEMM; the headline; SGEMM, CGEMM, ZGEMM x 4 transposes with K40c
    limits), with the host CPU model; N_space (the unpruned space, closed
    form) as context."""
    import beast_inputs as bi
    import oracle.closed_form
    cores = os.cpu_count() or 1
    d_all, pts, surv, dt = _oracle_run(desc, cores, 1e9)
    d1, pts1, _, dt1 = _oracle_run(desc, 1, budget_s)
    configs = []
    groups = [("configs[0] tiny DGEMM NN", [bi.tiny("D")]),
              ("configs[1] headline DGEMM NN K40c", [bi.headline()]),
              ("configs[2] S/C/Z x 4 transposes K40c",
               [bi.k40c(p, a, b) for p in ("S", "C", "Z") for a, b in bi.TRANSPOSES])]
    for name, spaces in groups:
        tot_p = tot_s = tot_t = 0.0
        for sp in spaces:
            _, p_, s_, t_ = _oracle_run(sp, cores, 1e9)
            tot_p += p_
            tot_s += s_
            tot_t += t_
        # one thread: the first space of the group, bounded
        dd, p1, _, t1 = _oracle_run(spaces[0], 1, budget_s / 2)
        configs.append({"config": name, "spaces": len(spaces), "points": int(tot_p), "survivors": int(tot_s),
                        "all_cores": {"s": tot_t, "points_per_s": tot_p / tot_t, "survivors_per_s": tot_s / tot_t},
                        "single_thread": {"s": t1, "points_per_s": p1 / t1,
                                          "sample": "whole first space" if dd is None else
                                          "first space, canonical prefix dim_m <= %d" % dd}})
    return {"value": pts / dt, "unit": UNIT, "cores": cores, "kind": "oracle",
            "sample": "whole %s space once (%d points, %.1f s wall on %d threads), canonical nest"
                      % (workload, pts, dt, cores),
            "survivors_per_s": surv / dt,
            "single_thread": {"value": pts1 / dt1, "unit": UNIT, "s": dt1,
                              "sample": "whole space" if d1 is None else "canonical prefix dim_m <= %d" % d1},
            "configs": configs, "cpu": _cpu_model(),
            "n_space": str(oracle.closed_form.n_space(desc)),
            "n_space_note": "size of the unpruned dependent-range space (closed form, context only; never a rate)"}


def relaunch(args):
    """`--gpus N` (N > 1) without a launcher: start N ranks on this node
    under torch.distributed.run (127.0.0.1) with this command line; rank 0
    prints the JSON line.  Fails (exit 2) if fewer than N GPUs are visible."""
    import socket
    try:
        import torch
        visible = torch.cuda.device_count()
    except Exception:
        visible = 0
    if visible < args.gpus:
        print("bench.py: --gpus %d but only %d CUDA device(s) visible; not measuring" % (args.gpus, visible),
              file=sys.stderr)
        return 2
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    env = dict(os.environ)
    env.setdefault("NCCL_DEBUG", "INFO")              # communicator / transport lines (NVLS, P2P) ...
    env.setdefault("NCCL_DEBUG_SUBSYS", "INIT")
    env.setdefault("NCCL_DEBUG_FILE", "/dev/stderr")  # ... on stderr, so stdout carries only the JSON line
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", str(args.gpus),
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd, env=env)


if __name__ == "__main__":
    sys.exit(main())

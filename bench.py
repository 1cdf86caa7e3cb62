#!/usr/bin/env python
"""bench.py -- FluidiCL on B200: end-to-end cooperative kernel time, roofline, oracle baseline.

Default workload (BASELINE.json configs[1]): GESUMMV + BICG (both kernels), N = 4096, fp32,
on one B200 plus the host cores.  One step = the three kernel launches through the C-ABI in
FluidiCL cooperative mode (GPU dispatcher + host executor + staging + diff-merge + return of
outputs), outputs coherent on the host at the end.  Inputs are resident in HBM and in the
pinned host mirrors when the timed region starts; L2 is flushed between steps.

Reported value: algorithmic GB/s of the step (bytes the kernels must move: every matrix
read once per kernel, vectors read/written) / device-timed step duration, summed over ranks.
Multi-GPU (torchrun): each rank runs an independent problem of the same size ("replicas",
weak scaling, no data-path collective); the max step time over ranks is used.  Every line also
carries `sharded_conv2d_corr`: BASELINE configs[3] (2DCONV 16384^2 + CORR 4096^2) sharded over
the same N ranks with NCCL all-gathers (strong scaling), so a 1/2/4/8-GPU run records both.

Also reported: GPU-only / CPU-only step times (the paper's two baselines, Fig 13), the merge
kernel's HBM bandwidth on a 1 GiB diff-merge, the dispatcher's roofline, the oracle timed
on the host cores (cpu_baseline) and an end-to-end number with the inputs' host->device
copies inside the timed region (e2e).

--impl reference times the oracle (the tier's reference arm) on the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np

METRIC = "end-to-end kernel time vs GPU-only/CPU-only; merge HBM GB/s vs peak"
N = 4096


def algorithmic_bytes(n: int) -> dict:
    f = 4
    return {
        "gesummv": 2 * n * n * f + 3 * n * f,   # A, B, x read; tmp, y written
        "bicg_s": n * n * f + 2 * n * f,        # A, r read; s written
        "bicg_q": n * n * f + 2 * n * f,        # A, p read; q written
    }


def problems(seed: int):
    import workloads as W
    P1 = W.make("gesummv", N, seed=seed, lws1d=256, out_init="zero")
    P2 = W.make("bicg_s", N, N, seed=seed + 1, lws1d=256, out_init="zero")
    P3 = W.make("bicg_q", N, N, seed=seed + 2, lws1d=256, out_init="zero")
    P3.bufs[0] = P2.bufs[0]          # BICG: both kernels read the same A
    return [P1, P2, P3]


# ---------------------------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi sampling clocks every 100 ms into a temporary file.  No Python thread reads
    its pipe: a reader thread competing for the GIL with the launching thread stalled
    cooperative steps by milliseconds."""

    def __init__(self, index: int, cores=None):
        self.index, self.proc, self.path, self.cores = index, None, None, cores

    def __enter__(self):
        if os.environ.get("FCL_NO_CLOCKS"):
            return self
        import tempfile
        q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            fd, self.path = tempfile.mkstemp(prefix="fcl_clocks_", suffix=".csv")
            self.out = os.fdopen(fd, "w")
            cores = self.cores
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={q}", "--format=csv,noheader,nounits",
                                          "-i", str(self.index), "-lms", "100"],
                                         stdout=self.out, stderr=subprocess.DEVNULL, text=True,
                                         # on the core(s) no host-executor thread spins on
                                         preexec_fn=(lambda: os.sched_setaffinity(0, cores)) if cores else None)
        except Exception:
            self.proc = None
        return self

    @property
    def lines(self) -> list:
        if not self.path:
            return []
        try:
            with open(self.path) as f:
                return [l.strip() for l in f if l.strip()]
        except OSError:
            return []

    def wait_started(self, timeout: float = 10.0):
        """Block until the sampler has printed its first sample: nvidia-smi's start-up (process
        spawn, NVML init) competes with the launch path for host cores and driver locks, so it
        must not fall inside the timed region."""
        t0 = time.perf_counter()
        while self.proc and not self.lines and time.perf_counter() - t0 < timeout:
            time.sleep(0.01)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=2)
            except Exception:
                self.proc.kill()
            self.out.close()

    def summary(self) -> dict:
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in list(self.lines):
            p = [x.strip() for x in l.split(",")]
            if len(p) < 9:
                continue
            try:
                sm.append(float(p[1])); mx = float(p[2])
            except ValueError:
                continue
            for nm, v in zip(names, p[5:9]):
                if v.lower() == "active":
                    reasons.add(nm)
        if self.path:
            try:
                os.unlink(self.path)
            except OSError:
                pass
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def measured_peaks() -> dict:
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return {"hbm_gbs": float(d["hbm_gbs"]), "source": "measured"}
    return {"hbm_gbs": 6650.0, "source": "fallback (B200_PROFILING.md)"}


def ncu_traffic(kernel: str):
    """DRAM bytes per launch of `kernel` from the committed ncu capture, or None."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        with open(p) as f:
            return json.load(f).get(kernel)
    return None


# ---------------------------------------------------------------------------------- oracle legs
def oracle_step_seconds(Ps, reps: int = 1) -> float:
    import oracle  # test infrastructure: only the cpu_baseline / --impl reference legs use it
    Ls = []
    for P in Ps:
        bufs = [b.astype(np.float64) for b in P.bufs]
        Ls.append(oracle.Launch(P.kernel, P.integer, P.n0, P.n1, list(P.gws), list(P.lws), bufs,
                                alpha=P.alpha, beta=P.beta))
    t0 = time.perf_counter()
    for _ in range(reps):
        for L in Ls:
            oracle.run_range(L, 0, L.num_groups())
    return (time.perf_counter() - t0) / reps


def run_reference(args, rank: int, world: int):
    if rank != 0:
        return
    Ps = problems(0)
    step_bytes = sum(algorithmic_bytes(N).values())
    for _ in range(args.warmup):
        oracle_step_seconds(Ps)
    times = [oracle_step_seconds(Ps) for _ in range(args.steps)]
    t = sum(times) / len(times)
    v = step_bytes / t / 1e9
    line = {"impl": "reference", "metric": METRIC, "value": round(v, 4), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t * 1e3, 3),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f64",
            "data": "synthetic",
            "config": {"workload": "gesummv_bicg4096", "n": N, "kernels": ["gesummv", "bicg_s", "bicg_q"]},
            "cpu_baseline": {"value": round(v, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                             "sample": "full step: serial C oracle (fp64) of GESUMMV + BICG s/q at N=4096"},
            "e2e": {"value": round(v, 4), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ---------------------------------------------------------------------------------- product leg
def run_fcl(args, rank: int, world: int, local_rank: int):
    import torch
    import fcl_harness as H
    from paper_conf_cgo_panditg14_b200 import _build, fcl

    if rank == 0:
        _build.build()
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    stream = torch.cuda.Stream(device=dev)
    # each local rank gets its own slice of the host cores (its host executor is pinned inside
    # it); within a slice one core is the coordinator's and one the caller's (runtime default)
    all_cores = sorted(os.sched_getaffinity(0))
    lws_ranks = max(1, int(os.environ.get("LOCAL_WORLD_SIZE", world)))
    per_rank = max(1, len(all_cores) // lws_ranks)
    if lws_ranks > 1:
        os.sched_setaffinity(0, all_cores[local_rank * per_rank:(local_rank + 1) * per_rank] or all_cores)
    cores = len(os.sched_getaffinity(0))
    # host executor threads: all cores but three -- the coordinator's, the caller's, and one
    # left free for the OS and the nvidia-smi clock sampler (a sampler that has to preempt a
    # spinning thread stalls the launch path by milliseconds)
    host_threads = max(1, cores - 3)
    ctx = fcl.Context(local_rank, n_host_threads=host_threads, streams=(stream.cuda_stream, None, None))
    # the launching thread on the core the runtime leaves for it; the clock sampler on the one
    # left free (coordinator, caller and workers take the others)
    slice_cores = H.pin_caller()
    free_cores = set(slice_cores[2 + host_threads:]) if slice_cores else None

    Ps = problems(1000 * rank)
    step_bytes = sum(algorithmic_bytes(N).values())
    # buffers: BICG's A shared by both kernels
    bufs = [H.create_buffers(ctx, Ps[0])]
    b2 = H.create_buffers(ctx, Ps[1])
    b3 = H.create_buffers(ctx, Ps[2])
    b3[0].release()
    b3[0] = b2[0]
    bufs += [b2, b3]
    prepared = {m: [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=m)
                    for P, b in zip(Ps, bufs)] for m in ("coop", "gpu", "cpu")}
    # the method without device selection: every launch runs cooperatively
    prepared["coop_always"] = [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode="coop",
                                           select=-1) for P, b in zip(Ps, bufs)]
    # per-launch detail steps only: CUDA timing events around the dominant kernel (GESUMMV).
    # Not in the timed steps -- a timing event between two grids keeps the second from
    # starting under the first's tail (programmatic dependent launch) and costs ~3 us itself.
    prepared["coop_t"] = [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode="coop",
                                      timing=(k == 0)) for k, (P, b) in enumerate(zip(Ps, bufs))]
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    # read sweep after the write flush: L2 ends full of clean, unrelated lines (no dirty
    # write-backs charged to the next kernel)
    sweep = torch.ones(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)

    def step(mode: str, infos: list = None):
        for launch in prepared[mode]:
            launch()
            if infos is not None:
                ctx.finish()
                infos.append(ctx.launch_info())
        ctx.finish()

    def one_step(mode: str, infos=None, idle=True) -> float:
        with torch.cuda.stream(stream):
            flush.fill_(1.0); sweep.sum()          # L2 flush (outside the timed interval)
        # idle GPU at e0: host-side work (the CPU-only leg, the host share of a cooperative
        # launch, launch submission) cannot hide under the flush.  The per-launch detail
        # steps (idle=False) instead queue behind the flush, so that the kernel-only events
        # see device time and not the host's submission latency.
        if idle:
            stream.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        step(mode, infos)
        e1.record(stream)
        e1.synchronize()
        return e0.elapsed_time(e1)

    def timed(mode: str, k: int, collect=False, idle=True):
        ts, infos = [], []
        for _ in range(k):
            ts.append(one_step(mode, infos if collect else None, idle))
        return ts, infos

    def timed_interleaved(modes, k: int):
        # the baselines step by step next to the measured mode: slow drifts of the host (PCIe,
        # clocks, the hypervisor) hit every mode alike; the order rotates every step, so that no
        # mode always follows the same one (a cooperative step's host side may still be winding
        # down when the next step starts)
        ts = {m: [] for m in modes}
        for r in range(k):
            for q in range(len(modes)):
                m = modes[(q + r) % len(modes)]
                ts[m].append(one_step(m))
        return ts

    def max_over_ranks(x: float) -> float:
        if dist is None:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    # warm-up (all modes), then the timed COOP steps
    for m in ("gpu", "cpu", "coop_always", "coop"):
        for _ in range(max(1, args.warmup)):
            step(m)
    if dist is not None:
        dist.barrier()
    torch.cuda.synchronize()
    import gc
    with ClockSampler(local_rank, free_cores or None) as clk:
        clk.wait_started()
        for _ in range(max(1, args.warmup)):   # re-warm after the sampler's start-up
            step("coop")
        if dist is not None:
            dist.barrier()
        torch.cuda.synchronize()
        gc.collect()
        gc.disable()   # as timeit does: no cyclic collection inside the timed region
        # one untimed step of every mode right before the timed ones: the first step after the
        # collection above runs cold (host caches, the pool of worker threads asleep) and would
        # otherwise always land on the first mode of the rotation
        for m in ("coop", "gpu", "coop_always"):
            one_step(m)
        c0 = ctx.counters()
        t_wall0 = time.perf_counter()
        # the timed COOP steps, each followed by a GPU-only step and a COOP step without device
        # selection (baselines under the same conditions: sampler running, gc off)
        tsm = timed_interleaved(("coop", "gpu", "coop_always"), args.steps)
        torch.cuda.synchronize()
        t_wall = time.perf_counter() - t_wall0
        c1 = ctx.counters()
        coop_ts, gpu_ts, always_ts = tsm["coop"], tsm["gpu"], tsm["coop_always"]
        gc.enable()
        if dist is not None:
            dist.barrier()
        # the timed region can be shorter than nvidia-smi's sampling period: keep the same
        # workload running (untimed) until the sampler has seen the clocks under this load
        t_s = time.perf_counter()
        while len(clk.lines) < 5 and time.perf_counter() - t_s < 3.0:
            step("coop")
    coop_ms = max_over_ranks(sum(coop_ts) / len(coop_ts))
    always_ms = max_over_ranks(sum(always_ts) / len(always_ts))
    # how the timed COOP launches ran (device selection); the coop_always steps
    # add only cooperative non-probe launches, the GPU-only steps only gpu_only
    dc = {k: c1[k] - c0[k] for k in c0}
    selection = {"launches": 3 * args.steps, "probes_cooperative": dc["probe"], "gpu_alone": dc["sel_gpu"],
                 "host_alone": dc["sel_cpu"], "select_period": "16, doubling up to 256 while probes confirm"}
    if os.environ.get("FCL_BENCH_DEBUG"):
        print("coop step ms:", [round(t, 3) for t in coop_ts], file=sys.stderr)

    # per-launch detail (dispatcher CUDA-event time, merges, host share) from separate steps
    _, infos = timed("coop_t", max(2, min(args.steps, 5)), collect=True, idle=False)
    gc.disable()
    cpu_ts, _ = timed("cpu", max(2, min(args.steps, 5)))
    gc.enable()
    gpu_ms = max_over_ranks(statistics.mean(gpu_ts))
    cpu_ms = max_over_ranks(statistics.mean(cpu_ts))
    ideal_ms = 1.0 / (1.0 / gpu_ms + 1.0 / cpu_ms)

    # dominant kernel: GESUMMV (2 N^2 floats); CUDA-event duration on main
    ges = infos[0::3]   # launch order per step: gesummv, bicg_s, bicg_q
    k_ms = statistics.mean(i["t_gpu_kernel_ms"] for i in ges if i["t_gpu_kernel_ms"] > 0)
    # which GPU path the COOP GESUMMV launches took (FCL_GPU_PATH_*): the GPU alone after device
    # selection (plain grid), the lite plain grid of a single-wave cooperative launch, or the
    # persistent dispatcher -- the first two run the same kernel
    paths = {i.get("gpu_path", 1) for i in ges}
    gesummv_kernel = ("coop_kernel<RowDotBody<float,2>> (GESUMMV dispatcher)" if 1 in paths
                      else "plain_kernel<RowDotBody<float,2>> (GESUMMV; COOP launch: lite grid or GPU alone "
                           "by device selection)")
    peaks = measured_peaks()
    achieved = algorithmic_bytes(N)["gesummv"] / (k_ms * 1e-3) / 1e9
    # Size ceiling: the same method MEASURED_PEAKS uses (torch copy, read + write bytes) at the
    # size of one GESUMMV launch (64 MiB copied = 134 MB moved), timed like the kernel (CUDA
    # events on the stream, queued behind the L2 flush).  A ~25 us kernel cannot reach the copy
    # peak measured on 2 GiB: launch, ramp and tail are a fixed few microseconds of it.
    # Context for `frac`, not a substitute for it.
    ceil_ts = []
    ra = torch.ones(N * N, dtype=torch.float32, device=dev)
    rb = torch.empty_like(ra)
    for r in range(8):
        with torch.cuda.stream(stream):
            flush.fill_(1.0); sweep.sum()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            rb.copy_(ra)
            e1.record(stream)
        e1.synchronize()
        if r >= 2:
            ceil_ts.append(e0.elapsed_time(e1))
    del ra, rb
    read_ceiling_gbs = 2 * N * N * 4 / (statistics.median(ceil_ts) * 1e-3) / 1e9
    # ... and torch's own read of the same bytes, GESUMMV's traffic pattern: one reduction over
    # 2 x 64 MiB (134 MB read, nothing written back) -- a reference point, not a ceiling (the
    # GESUMMV grid reads faster).  At this size a copy looks faster than a read: its 67 MB of
    # writes land in the 126 MB L2 and drain after the timed region.  The read ceiling of this
    # size, event-timed, is in profiles/r02_ubench_gesummv.txt (26.6 us, GESUMMV's pattern at it).
    ro_ts = []
    rr = torch.ones(2 * N * N, dtype=torch.float32, device=dev)
    for r in range(8):
        with torch.cuda.stream(stream):
            flush.fill_(1.0); sweep.sum()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            rr.sum()
            e1.record(stream)
        e1.synchronize()
        if r >= 2:
            ro_ts.append(e0.elapsed_time(e1))
    del rr
    readonly_ceiling_gbs = 2 * N * N * 4 / (statistics.median(ro_ts) * 1e-3) / 1e9
    launches_per_step = statistics.mean(
        sum(i["gpu_launches"] for i in infos[j:j + 3]) for j in range(0, len(infos) - 2, 3))

    # merge microbench: 1 GiB per stream, 10% of words changed (suffix), L2 flushed
    merge = None
    if rank == 0:
        nw = (1 << 30) // 4
        g = torch.randint(0, 2**31 - 1, (nw,), dtype=torch.int32, device=dev)
        t = torch.randint(0, 2**31 - 1, (nw,), dtype=torch.int32, device=dev)
        c = t.clone()
        c[-nw // 10:] ^= 1
        mts = []
        for r in range(8):
            with torch.cuda.stream(stream):
                flush.fill_(2.0); sweep.sum()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            fcl.merge_raw(g.data_ptr(), c.data_ptr(), t.data_ptr(), nw * 4, 4, stream.cuda_stream)
            e1.record(stream)
            e1.synchronize()
            if r >= 2:
                mts.append(e0.elapsed_time(e1))
        mms = statistics.median(mts)
        alg = nw * 8 + (nw // 10) * 4
        merge = {"bytes_per_stream": nw * 4, "changed_frac": 0.1, "ms": round(mms, 4),
                 "gbs": round(alg / (mms * 1e-3) / 1e9, 1),
                 "frac": round(alg / (mms * 1e-3) / 1e9 / peaks["hbm_gbs"], 4),
                 "traffic": ncu_traffic("merge_kernel")}
        del g, t, c

    # e2e: the same step with every input written from host memory (the pinned mirrors) and every
    # output read back, inside the timed region.  A non-blocking write of a whole buffer refreshes
    # the device copy lazily (include/fcl.h): with device selection the shapes whose inputs must
    # first cross PCIe are probed on their own, and run on the host alone when it covers the range
    # before the GPU got its data -- then nothing crosses PCIe.  The bytes actually moved are
    # counted by the runtime (fcl_get_counters); GPU-only mode is timed the same way beside it.
    in_bufs = [bufs[0][0], bufs[0][1], bufs[0][2], bufs[1][0], bufs[1][1], bufs[2][1]]
    out_bufs = [bufs[0][3], bufs[0][4], bufs[1][2], bufs[2][2]]
    in_bytes = sum(b.nbytes for b in in_bufs)
    out_bytes = sum(b.nbytes for b in out_bufs)
    outs = [np.empty(b.nbytes // 4, np.float32) for b in out_bufs]

    def e2e_step(mode):
        with torch.cuda.stream(stream):
            flush.fill_(3.0); sweep.sum()
        stream.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for b in in_bufs:
            b.write(b.host_ptr, blocking=False)     # host mirror -> (lazily) device
        step(mode)
        for b, o in zip(out_bufs, outs):
            b.read(o.ctypes.data)
        e1.record(stream)
        e1.synchronize()
        return e0.elapsed_time(e1)

    e2e_ts, e2e_gpu_ts = [], []
    for r in range(args.warmup):
        e2e_step("coop"); e2e_step("gpu")
    k0 = ctx.counters()
    for r in range(args.steps):
        e2e_ts.append(e2e_step("coop"))
    k1 = ctx.counters()
    for r in range(args.steps):
        e2e_gpu_ts.append(e2e_step("gpu"))
    e2e_ms = max_over_ranks(statistics.mean(e2e_ts))
    e2e_gpu_ms = max_over_ranks(statistics.mean(e2e_gpu_ts))
    e2e_h2d = (k1["h2d_bytes"] - k0["h2d_bytes"]) / args.steps
    e2e_d2h = (k1["d2h_bytes"] - k0["d2h_bytes"]) / args.steps
    e2e_sel = {"probes_cooperative": k1["probe"] - k0["probe"], "gpu_alone": k1["sel_gpu"] - k0["sel_gpu"],
               "host_alone": k1["sel_cpu"] - k0["sel_cpu"], "launches": 3 * args.steps}

    # oracle on the host cores (rank 0, N=1 only): one bounded full step
    cpu_baseline = None
    if rank == 0 and world == 1:
        t_or = oracle_step_seconds(problems(0))
        cpu_baseline = {"value": round(step_bytes / t_or / 1e9, 4), "unit": "GB/s", "cores": 1, "kind": "oracle",
                        "sample": f"one full step (GESUMMV + BICG s/q, N={N}) in the serial fp64 C oracle: "
                                  f"{t_or * 1e3:.0f} ms"}

    # BASELINE configs[3] at the same N, sharded over the ranks (strong scaling; the headline
    # `value` above is configs[1], one independent problem per rank): so that every line of a
    # 1/2/4/8-GPU scaling run also carries the sharded 2DCONV + CORR step with its NCCL exchanges
    sharded = None
    if os.environ.get("FCL_BENCH_SHARDED", "1") != "0":
        sharded = conv2d_corr_measure(max(2, min(args.steps, 10)), args.warmup, ctx, world, dev, stream, dist)

    if rank == 0:
        value = step_bytes * world / (coop_ms * 1e-3) / 1e9
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(coop_ms, 4), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": "gesummv_bicg4096", "n": N, "kernels": ["gesummv", "bicg_s", "bicg_q"],
                       "mode": "coop", "lws": 256, "work_groups_per_kernel": 16, "host_threads": host_threads,
                       "l2": "flushed between steps (256 MiB write + 256 MiB read sweep)", "parallelism": f"replicas{world}"},
            "coop_ms": round(coop_ms, 4), "coop_always_ms": round(always_ms, 4),
            "gpu_only_ms": round(gpu_ms, 4), "cpu_only_ms": round(cpu_ms, 4),
            "selection": selection,
            "ideal_coop_ms": round(ideal_ms, 4), "frac_of_ideal": round(ideal_ms / coop_ms, 4),
            "coop_vs_best_single": round(min(gpu_ms, cpu_ms) / coop_ms, 4),
            # (medians of the same interleaved steps: GPU-only and COOP-with-selection run the same
            # grids, so at 20 steps their means differ by the odd slow step of either)
            "median_ms": {"coop": round(statistics.median(coop_ts), 4), "gpu_only": round(statistics.median(gpu_ts), 4),
                          "coop_always": round(statistics.median(always_ts), 4)},
            "coop_vs_best_single_median": round(min(statistics.median(gpu_ts), cpu_ms) / statistics.median(coop_ts), 4),
            "wall_ms_per_step": round(t_wall * 1e3 / args.steps, 4),
            "roofline": {"kernel": gesummv_kernel, "bound": "hbm",
                         "achieved": round(achieved, 1), "peak": peaks["hbm_gbs"], "unit": "GB/s",
                         "frac": round(achieved / peaks["hbm_gbs"], 4), "traffic": ncu_traffic("gesummv"),
                         "algorithmic_bytes": algorithmic_bytes(N)["gesummv"], "kernel_ms": round(k_ms, 4),
                         "peak_source": peaks["source"],
                         "size_ceiling": {"what": "torch copy of 64 MiB (134 MB moved, as MEASURED_PEAKS but at this size), CUDA events, L2 flushed",
                                          "gbs": round(read_ceiling_gbs, 1),
                                          "achieved_over_ceiling": round(achieved / read_ceiling_gbs, 4),
                                          "torch_read": {"what": "torch sum over 2 x 64 MiB (134 MB read, one launch), CUDA events, L2 flushed; a reference point, not a ceiling",
                                                         "gbs": round(readonly_ceiling_gbs, 1),
                                                         "achieved_over": round(achieved / readonly_ceiling_gbs, 4)}}},
            "merge": merge,
            "cpu_baseline": cpu_baseline,
            "e2e": {"value": round(step_bytes * world / (e2e_ms * 1e-3) / 1e9, 3), "unit": "GB/s",
                    "ms_per_step": round(e2e_ms, 4), "h2d_bytes_per_step": int(round(e2e_h2d)),
                    "d2h_bytes_per_step": int(round(e2e_d2h)), "input_bytes_written_per_step": in_bytes,
                    "output_bytes_read_per_step": out_bytes, "selection": e2e_sel,
                    "gpu_only_ms_per_step": round(e2e_gpu_ms, 4),
                    "gpu_only_value": round(step_bytes * world / (e2e_gpu_ms * 1e-3) / 1e9, 3)},
            "gpu_launches": int(round(launches_per_step * args.steps)),
            "sharded_conv2d_corr": sharded,
            "clocks": clk.summary(),
            "host_cores": cores,
        }
        print(json.dumps(line), flush=True)
    ctx.release()


# ---------------------------------------------------------------------------------- config 4
CONV_N, CORR_N = 16384, 4096


def conv2d_corr_bytes() -> dict:
    """Algorithmic bytes of one config-4 step: 2DCONV reads A and writes B once; CORR mean/std read
    the data once, reduce reads and writes it, symmat reads its operand once (its roofline is FP32
    FFMA: its flops are M^2 N, reported separately)."""
    f, n, m = 4, CORR_N, CORR_N
    return {"conv2d": 2 * CONV_N * CONV_N * f, "corr_mean": n * m * f + m * f, "corr_std": n * m * f + 2 * m * f,
            "corr_reduce": 2 * n * m * f + 2 * m * f, "corr_corr": n * m * f + m * m * f}


def run_conv2d_corr(args, rank: int, world: int, local_rank: int):
    """BASELINE.json configs[3] on its own (`--workload conv2d_corr`): see conv2d_corr_measure."""
    import torch
    import fcl_harness as H
    from paper_conf_cgo_panditg14_b200 import _build, fcl
    if rank == 0:
        _build.build()
    dist = None
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    stream = torch.cuda.Stream(device=dev)
    all_cores = sorted(os.sched_getaffinity(0))
    lws_ranks = max(1, int(os.environ.get("LOCAL_WORLD_SIZE", world)))
    per_rank = max(1, len(all_cores) // lws_ranks)
    if lws_ranks > 1:
        os.sched_setaffinity(0, all_cores[local_rank * per_rank:(local_rank + 1) * per_rank] or all_cores)
    cores = len(os.sched_getaffinity(0))
    host_threads = max(1, cores - 3)
    ctx = fcl.Context(local_rank, n_host_threads=host_threads, streams=(stream.cuda_stream, None, None))
    H.pin_caller()
    with ClockSampler(local_rank) as clk:
        clk.wait_started()
        res = conv2d_corr_measure(args.steps, args.warmup, ctx, world, dev, stream, dist)
    if rank == 0:
        line = {"metric": METRIC, "value": res["value"], "unit": "GB/s", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["coop_ms"], "higher_is_better": True,
                "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": res["config"], "coop_ms": res["coop_ms"], "gpu_only_ms": res["gpu_only_ms"],
                "coop_vs_gpu_only": res["coop_vs_gpu_only"], "clocks": clk.summary(), "host_cores": cores}
        print(json.dumps(line), flush=True)
    ctx.release()


def conv2d_corr_measure(steps: int, warmup: int, ctx, world: int, dev, stream, dist) -> dict:
    """BASELINE.json configs[3]: 2DCONV 16384^2 and the CORR 4096^2 chain, the fixed problem sharded
    over the N ranks (strong scaling): each rank runs the cooperative path on its work-group
    slices with its own host pool, and every kernel's output is exchanged with an all-gather over
    NCCL into the ranks' device copies.  One step = both kernels' chains with their
    exchanges; the timed region covers the launches, the host sides and the collectives (CUDA
    events on the launching stream, max over ranks).  COOP and GPU-only steps alternate."""
    import torch
    import fcl_harness as H
    import workloads as W
    from paper_conf_cgo_panditg14_b200 import multigpu
    P = W.make("conv2d", CONV_N, CONV_N, seed=11, out_init="zero")
    A, B = H.create_buffers(ctx, P)
    n = m = CORR_N
    data0 = W.corr_chain_inputs(n, m, seed=12)
    gws1, lws1 = W.geometry("corr_mean", n, m, lws1d=256)
    gws2, lws2 = W.geometry("corr_reduce", n, m)
    d = ctx.buffer_from_array(data0)
    mean, std = ctx.buffer_from_array(np.zeros(m, np.float32)), ctx.buffer_from_array(np.zeros(m, np.float32))
    sym = ctx.buffer_from_array(np.zeros(m * m, np.float32))
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)

    def reset():
        # CORR's reduce works in place: both copies of the data back to the input (untimed)
        d.write(data0.ctypes.data, blocking=True)
        with torch.cuda.stream(stream):
            flush.fill_(1.0)
        stream.synchronize()

    def step(mode):
        with torch.cuda.stream(stream):
            multigpu.conv2d_sharded(ctx, A, B, P.n0, P.n1, P.gws, P.lws, mode=mode)
            multigpu.corr_sharded(ctx, d, mean, std, sym, n, m, gws1, lws1, gws2, lws2, mode=mode)

    def timed(mode):
        reset()
        if dist is not None:
            dist.barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        step(mode)
        e1.record(stream)
        e1.synchronize()
        t = e0.elapsed_time(e1)
        if dist is not None:
            x = torch.tensor([t], dtype=torch.float64, device=dev)
            dist.all_reduce(x, op=dist.ReduceOp.MAX)
            t = float(x.item())
        return t

    for _ in range(warmup):
        timed("coop"); timed("gpu")
    ts = {"coop": [], "gpu": []}
    for r in range(steps):
        for mode in (("coop", "gpu") if r % 2 == 0 else ("gpu", "coop")):
            ts[mode].append(timed(mode))
    coop_ms, gpu_ms = statistics.mean(ts["coop"]), statistics.mean(ts["gpu"])
    nbytes = sum(conv2d_corr_bytes().values())
    for b in (A, B, d, mean, std, sym):
        b.release()
    del flush
    return {"value": round(nbytes / (coop_ms * 1e-3) / 1e9, 2), "unit": "GB/s", "steps": steps,
            "coop_ms": round(coop_ms, 4), "gpu_only_ms": round(gpu_ms, 4),
            "coop_vs_gpu_only": round(gpu_ms / coop_ms, 4), "scaling": "strong",
            "config": {"workload": "conv2d_corr", "conv2d_n": CONV_N, "corr_n": CORR_N, "mode": "coop",
                       "parallelism": f"sharded{world} (work-group slices + NCCL all-gather)",
                       "l2": "flushed before each step (256 MiB write)",
                       "bytes_counted": "2DCONV 2 N^2 x 4 B; CORR mean/std/reduce data passes; symmat operand once"}}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="fcl", choices=["fcl", "reference"])
    ap.add_argument("--workload", default="gesummv_bicg4096", choices=["gesummv_bicg4096", "conv2d_corr"],
                    help="gesummv_bicg4096 (BASELINE configs[1], the headline; N > 1: replicas) or "
                         "conv2d_corr (configs[3]: one problem sharded over the ranks + NCCL all-gather)")
    args = ap.parse_args()
    args.warmup = max(3, args.warmup)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    if args.workload == "conv2d_corr":
        run_conv2d_corr(args, rank, world, local_rank)
    else:
        run_fcl(args, rank, world, local_rank)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()

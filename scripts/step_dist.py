"""Step-time distribution of the bench workload (GESUMMV + BICG 4096) per mode and host-thread
count: quantiles of CUDA-event step times, same flush/idle protocol as bench.py.  Diagnostic.

Usage: python scripts/step_dist.py [steps] [threads,...]
"""
import gc
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch

import bench
import fcl_harness as H
from paper_conf_cgo_panditg14_b200 import fcl

steps = int(sys.argv[1]) if len(sys.argv) > 1 else 200
thr = [int(x) for x in sys.argv[2].split(",")] if len(sys.argv) > 2 else [13]
if os.environ.get("SAMPLER"):   # an nvidia-smi clock sampler running alongside, as in bench.py
    import subprocess
    sampler = subprocess.Popen(["nvidia-smi", "--query-gpu=index,clocks.sm", "--format=csv,noheader", "-lms", "100"],
                               stdout=subprocess.DEVNULL, stderr=subprocess.DEVNULL)
    import time
    time.sleep(2.0)
dev = torch.device("cuda", 0)
stream = torch.cuda.Stream(device=dev)
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
sweep = torch.ones(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)


def q(ts):
    s = sorted(ts)
    return {"mean": round(statistics.mean(s), 4), "p10": round(s[len(s) // 10], 4), "p50": round(s[len(s) // 2], 4),
            "p90": round(s[9 * len(s) // 10], 4), "p99": round(s[min(len(s) - 1, 99 * len(s) // 100)], 4),
            "max": round(s[-1], 4)}


for T in thr:
    ctx = fcl.Context(0, n_host_threads=T, streams=(stream.cuda_stream, None, None))
    cfg = os.environ.get("CFG")
    if cfg:   # any scripts/bench_configs.py configuration
        sys.path.insert(0, os.path.join(ROOT, "scripts"))
        from bench_configs import cfg_problems
        Ps, meta = cfg_problems(cfg)
        bufs = [H.create_buffers(ctx, P) for P in Ps]
        for dl, db, sl, sb in meta.get("shared", []):
            if bufs[dl][db] is not bufs[sl][sb]:
                bufs[dl][db].release()
                bufs[dl][db] = bufs[sl][sb]
    else:
        Ps = bench.problems(0)
        bufs = [H.create_buffers(ctx, Ps[0])]
        b2 = H.create_buffers(ctx, Ps[1])
        b3 = H.create_buffers(ctx, Ps[2])
        b3[0].release()
        b3[0] = b2[0]
        bufs += [b2, b3]
    prepared = {m: [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=m)
                    for P, b in zip(Ps, bufs)] for m in ("coop", "gpu")}

    def step(m):
        for L in prepared[m]:
            L()
        ctx.finish()

    for m in ("gpu", "coop"):
        for _ in range(5):
            step(m)
    res = {}
    for m in ("gpu", "coop", "gpu", "coop"):
        ts = []
        gc.disable()
        for _ in range(steps):
            with torch.cuda.stream(stream):
                flush.fill_(1.0); sweep.sum()
            stream.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            step(m)
            e1.record(stream)
            e1.synchronize()
            ts.append(e0.elapsed_time(e1))
        if os.environ.get("SHOW_SLOW"):
            print(m, "slow steps:", [(k, round(t, 3)) for k, t in enumerate(ts) if t > 3 * sorted(ts)[len(ts) // 2]], flush=True)
        gc.enable()
        res.setdefault(m, []).append(q(ts))
    print(f"threads={T}", res, flush=True)
    ctx.release()

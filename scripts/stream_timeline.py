"""Device-side timeline of one bench step: a CUDA event is recorded on the main stream after
each launch, plus the kernel-only events of every launch (FCL_LAUNCH_TIMING), so each
launch's interval splits into kernel time and the gap before it.  Both modes, same buffers.
Usage: python scripts/stream_timeline.py [config]  (default gesummv_bicg4096)
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))

import time
import torch

import fcl_harness as H
from bench_configs import cfg_problems
from paper_conf_cgo_panditg14_b200 import fcl


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "gesummv_bicg4096"
    Ps, meta = cfg_problems(name)
    stream = torch.cuda.Stream()
    ctx = fcl.Context(0, streams=(stream.cuda_stream, None, None))
    bufs = [H.create_buffers(ctx, P) for P in Ps]
    for dl, db, sl, sb in meta.get("shared", []):
        bufs[dl][db] = bufs[sl][sb]
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    # read sweep after the write flush: L2 ends full of clean, unrelated lines (no dirty
    # write-backs charged to the next kernel)
    sweep = torch.ones(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    modes = ("gpu", "coop")
    Ls = {m: [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=m, timing=True)
              for P, b in zip(Ps, bufs)] for m in modes}
    iv = {m: [[] for _ in Ps] for m in modes}
    km = {m: [[] for _ in Ps] for m in modes}
    tail = {m: [] for m in modes}
    host = {m: [] for m in modes}
    reps = int(os.environ.get("REPS", "60"))
    for rep in range(reps + 5):
        for mode in modes:   # interleaved: slow drifts of the box hit both modes alike
            ctx.finish()
            with torch.cuda.stream(stream):
                flush.fill_(1.0); sweep.sum()
            stream.synchronize()
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(len(Ps) + 2)]
            t0 = time.perf_counter()
            ev[0].record(stream)
            for k, L in enumerate(Ls[mode]):
                L()
                ev[k + 1].record(stream)
            ctx.finish()
            ev[-1].record(stream)
            ev[-1].synchronize()
            t1 = time.perf_counter()
            if rep < 5:
                continue
            for k in range(len(Ps)):
                iv[mode][k].append(ev[k].elapsed_time(ev[k + 1]) * 1e3)
            tail[mode].append(ev[-2].elapsed_time(ev[-1]) * 1e3)
            host[mode].append((t1 - t0) * 1e6)
    for rep in range(20):   # kernel-only event times, one launch at a time (warm L2)
        for mode in modes:
            for k, L in enumerate(Ls[mode]):
                L()
                ctx.finish()
                km[mode][k].append(ctx.launch_info()["t_gpu_kernel_ms"] * 1e3)
    med = statistics.median
    for mode in modes:
        print(json.dumps({"mode": mode,
                          "interval_us": [round(med(x), 1) for x in iv[mode]],
                          "kernel_us_isolated": [round(med(x), 1) for x in km[mode]],
                          "after_last_us": round(med(tail[mode]), 1),
                          "step_event_us": round(med([sum(x) for x in zip(*iv[mode])]) + med(tail[mode]), 1),
                          "step_host_us": round(med(host[mode]), 1),
                          "step_host_p10_p90": [round(statistics.quantiles(host[mode], n=10)[0], 1),
                                                round(statistics.quantiles(host[mode], n=10)[-1], 1)]}), flush=True)
    ctx.release()


if __name__ == "__main__":
    main()

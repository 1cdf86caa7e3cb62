"""Dispatcher vs plain-grid time of ONE launch, two ways (CUDA events around the kernel):
  busy: the launch is queued behind an L2-flush kernel, so the events see device time only;
  idle: the stream is synchronized first, so the events also see the host submission latency.
Usage: python scripts/kernel_gap.py [config ...]   (configs of scripts/bench_configs.py; the
dominant launch of each is timed, earlier launches of the config run untimed first).
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))

import torch

import fcl_harness as H
from bench_configs import cfg_problems, algorithmic, HBM, FP32_TFLOPS
from paper_conf_cgo_panditg14_b200 import fcl


def main():
    names = sys.argv[1:] or ["gesummv_bicg4096", "syrk2048", "syr2k2048", "conv2d16384"]
    for name in names:
        Ps, meta = cfg_problems(name)
        stream = torch.cuda.Stream()
        ctx = fcl.Context(0, streams=(stream.cuda_stream, None, None))
        bufs = [H.create_buffers(ctx, P) for P in Ps]
        for dl, db, sl, sb in meta.get("shared", []):
            bufs[dl][db] = bufs[sl][sb]
        dom = max(range(len(Ps)), key=lambda k: algorithmic(Ps[k])[1] / (HBM * 1e9 if algorithmic(Ps[k])[0] == "hbm" else FP32_TFLOPS * 1e12))
        flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
        # read sweep after the write flush: L2 ends full of clean, unrelated lines (no dirty
        # write-backs charged to the next kernel)
        sweep = torch.ones(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
        out = {"config": name, "kernel": H.kernel_name(Ps[dom])}
        reps = 12 if name not in ("conv2d16384",) else 4
        for mode in ("gpu", "coop"):
            L = ctx.prepare(H.kernel_name(Ps[dom]), Ps[dom].gws, Ps[dom].lws, H.make_args(ctx, Ps[dom], bufs[dom]),
                            mode=mode, timing=True)
            for regime in ("busy", "idle"):
                ts = []
                for r in range(reps + 2):
                    ctx.finish()
                    with torch.cuda.stream(stream):
                        flush.fill_(1.0); sweep.sum()
                    if regime == "idle":
                        stream.synchronize()
                    L()
                    ctx.finish()
                    if r >= 2:
                        ts.append(ctx.launch_info()["t_gpu_kernel_ms"])
                out[f"{mode}_{regime}_ms"] = round(statistics.median(ts), 4)
        print(json.dumps(out), flush=True)
        ctx.release()


if __name__ == "__main__":
    main()

"""CUDA-event time of single GPU-only launches (the plain grid) after an L2 flush, median of 15,
with the algorithmic HBM fraction -- for A/B builds of one body.

Usage: python scripts/kernel_time.py kernel:n0:n1:lws [...]   e.g. bicg_s:4096:4096:256
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch

import fcl_harness as H
import workloads as W
from paper_conf_cgo_panditg14_b200 import fcl

PEAK = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0


def alg_bytes(P):
    return sum(b.nbytes for b in P.bufs)   # every buffer read or written once (dot kernels)


def main():
    stream = torch.cuda.Stream()
    ctx = fcl.Context(0, streams=(stream.cuda_stream, None, None))
    flush = torch.empty(256 << 18, dtype=torch.float32, device="cuda")
    # bench.py's flush: a write sweep, then a read sweep (L2 left full of clean lines, so the
    # timed kernel pays no write-backs of the flush)
    sweep = torch.ones(256 << 18, dtype=torch.float32, device="cuda")
    for spec in sys.argv[1:]:
        k, n0, n1, lws = spec.split(":")
        P = W.make(k, int(n0), int(n1), seed=0, lws1d=int(lws), out_init="zero")
        bufs = H.create_buffers(ctx, P)
        L = ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, bufs), mode="gpu", timing=1)
        ts = []
        for r in range(20):
            with torch.cuda.stream(stream):
                flush.fill_(float(r)); sweep.sum()
            L()
            ctx.finish()
            if r >= 5:
                ts.append(ctx.launch_info()["t_gpu_kernel_ms"])
        ms = statistics.median(ts)
        gbs = alg_bytes(P) / (ms * 1e-3) / 1e9
        print(json.dumps({"kernel": spec, "ms": round(ms, 4), "gbs": round(gbs, 1), "frac": round(gbs / PEAK, 4)}), flush=True)
        for b in bufs:
            b.release()
    ctx.release()


if __name__ == "__main__":
    main()

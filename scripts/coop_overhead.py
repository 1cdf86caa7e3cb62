"""Cooperative-step overhead vs GPU-only, bench-style timing (L2 flushed, idle GPU at e0, CUDA
events on the launching stream), COOP and GPU-only steps interleaved so that drift cancels.
Usage: python scripts/coop_overhead.py [config] [steps] [host_threads]
Prints one JSON line: medians / means of both modes and their difference.
"""
import gc
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))

import torch

import fcl_harness as H
from bench_configs import cfg_problems
from paper_conf_cgo_panditg14_b200 import fcl


def main():
    name = sys.argv[1] if len(sys.argv) > 1 else "gesummv_bicg4096"
    steps = int(sys.argv[2]) if len(sys.argv) > 2 else 200
    nthr = int(sys.argv[3]) if len(sys.argv) > 3 else max(1, len(os.sched_getaffinity(0)) - 3)
    Ps, meta = cfg_problems(name)
    stream = torch.cuda.Stream()
    ctx = fcl.Context(0, n_host_threads=nthr, streams=(stream.cuda_stream, None, None))
    H.pin_caller()
    bufs = [H.create_buffers(ctx, P) for P in Ps]
    for dl, db, sl, sb in meta.get("shared", []):
        bufs[dl][db] = bufs[sl][sb]
    prep = {m: [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=m)
                for P, b in zip(Ps, bufs)] for m in ("coop", "gpu")}
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    sweep = torch.ones_like(flush)

    def one(mode):
        with torch.cuda.stream(stream):
            flush.fill_(1.0); sweep.sum()
        stream.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for L in prep[mode]:
            L()
        ctx.finish()
        e1.record(stream)
        e1.synchronize()
        return e0.elapsed_time(e1)

    for _ in range(10):
        one("gpu"); one("coop")
    gc.collect(); gc.disable()
    ts = {"coop": [], "gpu": []}
    for _ in range(steps):
        for m in ("coop", "gpu"):
            ts[m].append(one(m))
    gc.enable()
    out = {"config": name, "host_threads": nthr, "env": {k: v for k, v in os.environ.items() if k.startswith("FCL_")}}
    for m, v in ts.items():
        out[m] = {"median": round(statistics.median(v), 4), "mean": round(statistics.mean(v), 4),
                  "p90": round(sorted(v)[int(0.9 * len(v))], 4), "min": round(min(v), 4)}
    out["coop_slowest"] = sorted(((round(t, 4), i) for i, t in enumerate(ts["coop"])), reverse=True)[:5]
    out["coop_vs_gpu_mean"] = round(out["gpu"]["mean"] / out["coop"]["mean"], 4)
    out["coop_vs_gpu_median"] = round(out["gpu"]["median"] / out["coop"]["median"], 4)
    print(json.dumps(out), flush=True)
    ctx.release()


if __name__ == "__main__":
    main()

"""Does BICG q find the matrix BICG s just read in L2?  CUDA-event time of each kernel of the
headline step (GPU-only plain grids, N = 4096), the step starting after an L2 flush, with and
without a second flush between bicg_s and bicg_q.  Median of 15.

Usage: python scripts/l2_reuse.py
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch

import bench
import fcl_harness as H
from paper_conf_cgo_panditg14_b200 import fcl


def main():
    stream = torch.cuda.Stream()
    ctx = fcl.Context(0, streams=(stream.cuda_stream, None, None))
    Ps = bench.problems(0)
    bufs = [H.create_buffers(ctx, Ps[0])]
    b2 = H.create_buffers(ctx, Ps[1])
    b3 = H.create_buffers(ctx, Ps[2])
    b3[0].release()
    b3[0] = b2[0]
    bufs += [b2, b3]
    L = [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode="gpu", timing=1)
         for P, b in zip(Ps, bufs)]
    flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")
    for mid_flush in (False, True):
        ts = [[], [], []]
        for r in range(20):
            for k in range(3):
                if k == 0 or (k == 2 and mid_flush):
                    with torch.cuda.stream(stream):
                        flush.fill_(float(r))
                L[k]()
                ctx.finish()
                if r >= 5:
                    ts[k].append(ctx.launch_info()["t_gpu_kernel_ms"])
        print(json.dumps({"flush_between_s_and_q": mid_flush,
                          "ms": {n: round(statistics.median(t), 4) for n, t in zip(("gesummv", "bicg_s", "bicg_q"), ts)}}),
              flush=True)
    ctx.release()


if __name__ == "__main__":
    main()

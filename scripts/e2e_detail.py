"""Where bench.py's e2e step (GESUMMV + BICG s/q, N = 4096, inputs written from host memory every
step) spends its time: per-kernel device assignments timed as whole steps, and one detailed step
per assignment (per-launch launch_info, a finish after each launch).

Usage: python scripts/e2e_detail.py [steps]
Prints one JSON line per assignment: {"modes": [...], "ms": mean, "median": ..., "h2d": bytes per
step, "detail": [per-launch info]}.
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import bench
import fcl_harness as H
from paper_conf_cgo_panditg14_b200 import fcl

KEYS = ("selected", "probe", "gpu_path", "cpu_wgs", "streamed_wgs", "h2d_bytes", "t_call_ms", "t_host_ms",
        "t_gpu_kernel_ms", "merged", "cpu_did_all")


def main():
    steps = int(sys.argv[1]) if len(sys.argv) > 1 else 10
    stream = torch.cuda.Stream()
    cores = len(os.sched_getaffinity(0))
    ctx = fcl.Context(0, n_host_threads=max(1, cores - 3), streams=(stream.cuda_stream, None, None))
    H.pin_caller()
    Ps = bench.problems(0)
    bufs = [H.create_buffers(ctx, Ps[0])]
    b2 = H.create_buffers(ctx, Ps[1])
    b3 = H.create_buffers(ctx, Ps[2])
    b3[0].release()
    b3[0] = b2[0]
    bufs += [b2, b3]
    in_bufs = [bufs[0][0], bufs[0][1], bufs[0][2], bufs[1][0], bufs[1][1], bufs[2][1]]
    out_bufs = [bufs[0][3], bufs[0][4], bufs[1][2], bufs[2][2]]
    outs = [np.empty(b.nbytes // 4, np.float32) for b in out_bufs]
    flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")

    def prep(modes, select):
        return [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=m,
                            **({} if select else {"select": -1}))
                for P, b, m in zip(Ps, bufs, modes)]

    def step(launches, detail=None):
        with torch.cuda.stream(stream):
            flush.fill_(3.0)
        stream.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for b in in_bufs:
            b.write(b.host_ptr, blocking=False)
        for L in launches:
            L()
            if detail is not None:
                ctx.finish()
                i = ctx.launch_info()
                detail.append({k: (round(i[k], 4) if isinstance(i[k], float) else i[k]) for k in KEYS})
        ctx.finish()
        for b, o in zip(out_bufs, outs):
            b.read(o.ctypes.data)
        e1.record(stream)
        e1.synchronize()
        return e0.elapsed_time(e1)

    cases = [(("gpu", "gpu", "gpu"), False), (("coop", "coop", "coop"), True), (("coop", "coop", "coop"), False),
             (("cpu", "cpu", "cpu"), False), (("cpu", "gpu", "gpu"), False), (("coop", "cpu", "coop"), False),
             (("cpu", "coop", "coop"), False), (("coop", "gpu", "gpu"), False), (("cpu", "cpu", "coop"), False),
             (("coop", "cpu", "cpu"), False), (("gpu", "cpu", "cpu"), False)]
    for modes, select in cases:
        L = prep(modes, select)
        for _ in range(3):
            step(L)
        c0 = ctx.counters()
        ts = [step(L) for _ in range(steps)]
        c1 = ctx.counters()
        det = []
        step(L, det)
        print(json.dumps({"modes": modes, "select": select, "ms": round(statistics.mean(ts), 4),
                          "median": round(statistics.median(ts), 4),
                          "h2d": (c1["h2d_bytes"] - c0["h2d_bytes"]) // steps, "detail": det}), flush=True)
    ctx.release()


if __name__ == "__main__":
    main()

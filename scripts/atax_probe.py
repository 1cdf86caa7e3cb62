"""ATAX 256 (BASELINE configs[0]): every per-kernel device assignment timed as whole steps (CUDA
events, idle GPU at the start, inputs resident), and the cooperative probes' outcomes per kernel
(host share, who finished first, chunk sizes).

Usage: python scripts/atax_probe.py [steps]
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
from bench_configs import cfg_problems
from paper_conf_cgo_panditg14_b200 import fcl

KEYS = ("selected", "probe", "gpu_path", "cpu_wgs", "cpu_did_all", "published_watermark", "n_chunks", "t_host_ms",
        "t_call_ms")


def main():
    steps = int(sys.argv[1]) if len(sys.argv) > 1 else 40
    Ps, meta = cfg_problems("atax256")
    stream = torch.cuda.Stream()
    ctx = fcl.Context(0, streams=(stream.cuda_stream, None, None))
    H.pin_caller()
    bufs = [H.create_buffers(ctx, P) for P in Ps]
    for (dl, db, sl, sb) in meta["shared"]:
        bufs[dl][db].release()
        bufs[dl][db] = bufs[sl][sb]
    flush = torch.empty(64 << 20, dtype=torch.float32, device="cuda")

    def prep(modes, select):
        return [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=m, select=select)
                for P, b, m in zip(Ps, bufs, modes)]

    def step(L, detail=None):
        with torch.cuda.stream(stream):
            flush.fill_(1.0)
        stream.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for launch in L:
            launch()
            if detail is not None:
                ctx.finish()
                i = ctx.launch_info()
                d = {k: (round(i[k], 4) if isinstance(i[k], float) else i[k]) for k in KEYS}
                d["chunks"] = list(i.get("chunk_sizes", []))
                detail.append(d)
        ctx.finish()
        e1.record(stream)
        e1.synchronize()
        return e0.elapsed_time(e1)

    cases = [(("cpu", "cpu"), 0), (("gpu", "gpu"), 0), (("cpu", "gpu"), 0), (("gpu", "cpu"), 0),
             (("coop", "coop"), -1), (("coop", "coop"), 1)]
    for modes, select in cases:
        L = prep(modes, select)
        for _ in range(5):
            step(L)
        c0 = ctx.counters()
        ts = [step(L) for _ in range(steps)]
        c1 = ctx.counters()
        det = []
        step(L, det)
        print(json.dumps({"modes": modes, "select": select, "ms": round(statistics.mean(ts), 4),
                          "median": round(statistics.median(ts), 4),
                          "counters": {k: c1[k] - c0[k] for k in ("probe", "sel_gpu", "sel_cpu")},
                          "detail": det}), flush=True)
    ctx.release()


if __name__ == "__main__":
    main()

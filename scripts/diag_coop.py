"""Diagnostics: per-launch breakdown of cooperative vs GPU-only execution (not a benchmark)."""
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np

import fcl_harness as H
import workloads as W
from paper_conf_cgo_panditg14_b200 import fcl


def main():
    kern = sys.argv[1] if len(sys.argv) > 1 else "gesummv"
    n = int(sys.argv[2]) if len(sys.argv) > 2 else 4096
    for status in ("host_mapped", "device"):
        ctx = fcl.Context(0, status_location=status)
        if kern in ("syrk", "syr2k", "conv2d", "corr_reduce"):
            P = W.make(kern, n, n, seed=0, out_init="zero")
        else:
            P = W.make(kern, n, n, seed=0, lws1d=256, out_init="zero")
        bufs = H.create_buffers(ctx, P)
        args = H.make_args(ctx, P, bufs)
        name = H.kernel_name(P)
        configs = [("gpu", {}), ("coop", dict(forced_split=P.num_groups)), ("coop", dict(drop_publish=1)),
                   ("coop", dict(n_host_threads=1)), ("coop", {}), ("cpu", {})]
        for mode, kw in configs:
            rows = []
            for rep in range(6):
                t0 = time.perf_counter()
                ctx.enqueue_ndrange(name, P.gws, P.lws, args, mode=mode, **kw)
                ctx.finish()
                t1 = time.perf_counter()
                info = ctx.launch_info()
                rows.append((t1 - t0) * 1e3)
            keep = {k: info[k] for k in ("gpu_watermark", "published_watermark", "gpu_tasks", "gpu_tasks_total",
                                         "cpu_wgs", "n_chunks", "cpu_did_all", "merged", "t_gpu_kernel_ms",
                                         "t_merge_ms", "t_host_ms", "t_call_ms", "chunk_sizes")}
            print(json.dumps({"status": status, "mode": mode, "opts": kw, "wall_ms_med": round(float(np.median(rows[1:])), 4),
                              **keep}), flush=True)
        for b in bufs:
            b.release()
        ctx.release()


if __name__ == "__main__":
    main()

"""Bench-like steps (L2 flush on the main stream before each step) with per-launch info."""
import json
import os
import sys

os.environ.setdefault("FCL_TRACE", "1")
os.environ.setdefault("FCL_STATS", "1")
os.environ.setdefault("FCL_TRACE_FILE", "gpurun_out/trace_b.txt")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch
import fcl_harness as H
import workloads as W
from paper_conf_cgo_panditg14_b200 import fcl

flush_on = int(sys.argv[1]) if len(sys.argv) > 1 else 1
stream = torch.cuda.Stream()
ctx = fcl.Context(0, streams=(stream.cuda_stream, None, None))
Ps = [W.make("gesummv", 4096, seed=0, lws1d=256, out_init="zero"),
      W.make("bicg_s", 4096, 4096, seed=1, lws1d=256, out_init="zero"),
      W.make("bicg_q", 4096, 4096, seed=2, lws1d=256, out_init="zero")]
launches = []
for P in Ps:
    b = H.create_buffers(ctx, P)
    launches.append(ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode="coop"))
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
times = []
for rep in range(20):
    if flush_on:
        with torch.cuda.stream(stream):
            flush.fill_(1.0)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    infos = []
    for L in launches:
        L()
    ctx.finish()
    e1.record(stream)
    e1.synchronize()
    times.append(e0.elapsed_time(e1))
print("step ms:", [round(t, 3) for t in times[-8:]])
for L in launches:
    L()
    ctx.finish()
    i = ctx.launch_info()
    print(json.dumps({k: i[k] for k in ("gpu_watermark", "published_watermark", "cpu_wgs", "n_chunks", "merged",
                                         "gpu_launches", "t_gpu_kernel_ms", "t_host_ms", "chunk_sizes", "h2d_bytes",
                                         "d2h_bytes")}))
ctx.release()
recs = [l.split() for l in open(os.environ["FCL_TRACE_FILE"])]
steps, cur = [], []
for t, tag, e in recs:
    if tag.startswith("gpu_"):
        continue
    cur.append((float(t), tag, int(e)))
    if tag == "finish_end":
        steps.append(cur); cur = []
for st in steps[-24:-22]:
    t0 = st[0][0]
    print(" | ".join(f"{tag}:{e}@{(t - t0) * 1000:.1f}us" for t, tag, e in st))

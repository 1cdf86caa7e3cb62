"""Host-side trace of bench-like steps (FCL_TRACE=1): prints per-event offsets within each step."""
import os
import sys
import time

os.environ.setdefault("FCL_TRACE", "1")
os.environ.setdefault("FCL_STATS", "1")
os.environ.setdefault("FCL_TRACE_FILE", "gpurun_out/trace.txt")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import fcl_harness as H
import workloads as W
from paper_conf_cgo_panditg14_b200 import fcl

mode = sys.argv[1] if len(sys.argv) > 1 else "coop"
which = sys.argv[2] if len(sys.argv) > 2 else "gesummv_bicg4096"
sys.path.insert(0, os.path.join(ROOT, "scripts"))
from bench_configs import cfg_problems
ctx = fcl.Context(0)
Ps, meta = cfg_problems(which)
bufs = [H.create_buffers(ctx, P) for P in Ps]
for dl, db, sl, sb in meta.get("shared", []):
    bufs[dl][db] = bufs[sl][sb]
launches = [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=mode) for P, b in zip(Ps, bufs)]
flush = None
if os.environ.get("TRACE_FLUSH"):   # bench-like: L2 flushed and the GPU idle before each step
    import torch
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    sweep = torch.ones(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
for rep in range(30):
    if flush is not None:
        flush.fill_(1.0); sweep.sum()
        torch.cuda.synchronize()
    for L in launches:
        L()
    ctx.finish()
ctx.release()
# summarize the last steps: host events per step, device stamps separately
recs = [l.split() for l in open(os.environ["FCL_TRACE_FILE"])]
host = [(float(t), tag, int(e)) for t, tag, e in recs if not tag.startswith("gpu_")]
steps, cur = [], []
for t, tag, e in host:
    cur.append((t, tag, e))
    if tag == "finish_end":
        steps.append(cur); cur = []
show = steps[-3:]
if os.environ.get("TRACE_SLOWEST"):   # the slowest steps instead of the last ones
    show = sorted(steps, key=lambda st: st[-1][0] - st[0][0])[-int(os.environ["TRACE_SLOWEST"]):]
for st in show:
    t0 = st[0][0]
    print(" | ".join(f"{tag}:{e}@{(t - t0) * 1000:.1f}" for t, tag, e in st))
gpu = sorted((float(t), tag, int(e)) for t, tag, e in recs if tag.startswith("gpu_"))
if gpu:
    # device stamps of the last few slots, relative to the earliest of them (us)
    by_slot = {}
    for t, tag, e in gpu:
        by_slot.setdefault(e, {})[tag] = t
    last = sorted(by_slot.items(), key=lambda kv: min(kv[1].values()))[-6:]
    g0 = min(last[0][1].values())
    for slot, d in last:
        print("GPU slot", slot, " ".join(f"{k[4:-3]}@{(v - g0) * 1000:.1f}" for k, v in sorted(d.items(), key=lambda kv: kv[1])))

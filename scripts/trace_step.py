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
for rep in range(30):
    for L in launches:
        L()
    ctx.finish()
ctx.release()
# summarize the last 10 steps
recs = [l.split() for l in open(os.environ["FCL_TRACE_FILE"])]
steps, cur = [], []
for t, tag, e in recs:
    cur.append((float(t), tag, int(e)))
    if tag == "finish_end":
        steps.append(cur); cur = []
for st in steps[-3:]:
    t0 = st[0][0]
    print(" | ".join(f"{tag}:{e}@{(t - t0) * 1000:.1f}us" for t, tag, e in st))
gpu = [(float(t), tag, int(e)) for t, tag, e in recs if tag.startswith("gpu_")]
# last 6 slots' device stamps, relative to the earliest shown
gpu = sorted(gpu)[-12:]
if gpu:
    g0 = gpu[0][0]
    print("GPU:", " | ".join(f"{tag}[slot{e}]@{(t - g0) * 1000:.1f}us" for t, tag, e in gpu))

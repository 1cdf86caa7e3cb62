"""Host-side trace (FCL_TRACE=1) of interleaved steps, e.g. "gpu,coop,coop_always": prints the
event offsets of the last steps of the mode given last (bench-like: L2 flushed, idle GPU)."""
import os
import sys

os.environ.setdefault("FCL_TRACE", "1")
os.environ.setdefault("FCL_TRACE_FILE", "gpurun_out/trace_seq.txt")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
import torch

import fcl_harness as H
from bench_configs import cfg_problems
from paper_conf_cgo_panditg14_b200 import fcl

seq = (sys.argv[1] if len(sys.argv) > 1 else "gpu,coop,coop_always").split(",")
which = sys.argv[2] if len(sys.argv) > 2 else "gesummv_bicg4096"
stream = torch.cuda.Stream()
ctx = fcl.Context(0, n_host_threads=13, streams=(stream.cuda_stream, None, None))
H.pin_caller()
Ps, meta = cfg_problems(which)
bufs = [H.create_buffers(ctx, P) for P in Ps]
for dl, db, sl, sb in meta.get("shared", []):
    bufs[dl][db] = bufs[sl][sb]
prep = {}
for m in set(seq):
    mode, sel = ("coop", -1) if m == "coop_always" else (m, 0)
    prep[m] = [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=mode, select=sel)
               for P, b in zip(Ps, bufs)]
flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
sweep = torch.ones_like(flush)
times = {m: [] for m in seq}
for rep in range(40):
    for m in seq:
        with torch.cuda.stream(stream):
            flush.fill_(1.0); sweep.sum()
        stream.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for L in prep[m]:
            L()
        ctx.finish()
        e1.record(stream)
        e1.synchronize()
        times[m].append(e0.elapsed_time(e1))
ctx.release()
for m, v in times.items():
    print(m, "median ms", sorted(v)[len(v) // 2], "last", [round(x, 4) for x in v[-6:]])
recs = [l.split() for l in open(os.environ["FCL_TRACE_FILE"])]
host = [(float(t), tag, int(e)) for t, tag, e in recs if not tag.startswith("gpu_")]
steps, cur = [], []
for t, tag, e in host:
    cur.append((t, tag, e))
    if tag == "finish_end":
        steps.append(cur); cur = []
# the slowest steps of the last mode in the sequence (TRACE_LAST=1: its last steps)
k = len(seq)
mine = steps[k - 1::k]
show = mine[-3:] if os.environ.get("TRACE_LAST") else sorted(mine, key=lambda st: st[-1][0] - st[0][0])[-3:]
for st in show:
    t0 = st[0][0]
    print(" | ".join(f"{tag}:{e}@{(t - t0) * 1000:.1f}" for t, tag, e in st))

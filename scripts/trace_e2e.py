"""Host-side trace (FCL_TRACE=1) of the bench's e2e step: inputs written non-blocking (lazy device
refresh), three COOP launches, outputs read back.  Prints step times and the last step's events,
then per-launch info of one instrumented step (a finish after each launch)."""
import os
import sys

os.environ.setdefault("FCL_TRACE", "1")
os.environ.setdefault("FCL_TRACE_FILE", "gpurun_out/trace_e2e.txt")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))
import numpy as np
import torch

import fcl_harness as H
from bench_configs import cfg_problems
from paper_conf_cgo_panditg14_b200 import fcl

stream = torch.cuda.Stream()
ctx = fcl.Context(0, n_host_threads=13, streams=(stream.cuda_stream, None, None))
H.pin_caller()
Ps, meta = cfg_problems("gesummv_bicg4096")
bufs = [H.create_buffers(ctx, P) for P in Ps]
for dl, db, sl, sb in meta.get("shared", []):
    bufs[dl][db] = bufs[sl][sb]
L = [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode="coop") for P, b in zip(Ps, bufs)]
in_bufs = [bufs[0][0], bufs[0][1], bufs[0][2], bufs[1][0], bufs[1][1], bufs[2][1]]
out_bufs = [bufs[0][3], bufs[0][4], bufs[1][2], bufs[2][2]]
outs = [np.empty(b.nbytes // 4, np.float32) for b in out_bufs]
ts = []
import traceback
failed = False
for r in range(40):
  try:
      stream.synchronize()
      e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
      e0.record(stream)
      for b in in_bufs:
          b.write(b.host_ptr, blocking=False)
      for l in L:
          l()
      ctx.finish()
      for b, o in zip(out_bufs, outs):
          b.read(o.ctypes.data)
      e1.record(stream)
      e1.synchronize()
      ts.append(e0.elapsed_time(e1))
  except Exception:
    traceback.print_exc()
    print("FAILED at step", r)
    failed = True
    break
print("step ms", [round(t, 3) for t in ts[-12:]])
if failed:
    try:
        ctx.release()
    except Exception:
        pass
    recs = [l.split() for l in open(os.environ["FCL_TRACE_FILE"])]
    host = [(float(t), tag, int(e)) for t, tag, e in recs if not tag.startswith("gpu_")]
    t0 = host[-60][0] if len(host) > 60 else host[0][0]
    print(" | ".join(f"{tag}:{e}@{(t - t0) * 1000:.0f}" for t, tag, e in host[-60:]))
    sys.exit(1)
for b in in_bufs:
    b.write(b.host_ptr, blocking=False)
for l, P in zip(L, Ps):
    l()
    ctx.finish()
    i = ctx.launch_info()
    print(P.kernel, {k: i[k] for k in ("selected", "probe", "gpu_path", "cpu_wgs", "n_wg", "streamed_wgs", "h2d_bytes",
                                     "d2h_bytes", "cpu_did_all", "t_host_ms", "chunk_sizes")})
ctx.release()
recs = [l.split() for l in open(os.environ["FCL_TRACE_FILE"])]
host = [(float(t), tag, int(e)) for t, tag, e in recs if not tag.startswith("gpu_")]
steps, cur = [], []
for t, tag, e in host:
    cur.append((t, tag, e))
    if tag == "finish_end":
        steps.append(cur); cur = []
for st in steps[-6:-3]:
    t0 = st[0][0]
    print(" | ".join(f"{tag}:{e}@{(t - t0) * 1000:.0f}" for t, tag, e in st))

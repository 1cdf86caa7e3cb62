"""Stress loop of the e2e step (non-blocking input writes, streamed COOP launches with selection,
finish, reads) at N=1024: prints the step of the first failure.  Usage: python scripts/e2e_loop_stress.py STEPS"""
import os, sys, time
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import numpy as np
import fcl_harness as H
import workloads as W
from paper_conf_cgo_panditg14_b200 import fcl
ctx = fcl.Context(0)
Ps = [W.make("gesummv", 1024, seed=41, lws1d=64), W.make("bicg_s", 1024, 1024, seed=42, lws1d=64), W.make("bicg_q", 1024, 1024, seed=43, lws1d=64)]
bufs = [H.create_buffers(ctx, P) for P in Ps]
steps = int(sys.argv[1])
t0 = time.time()
for step in range(steps):
    for P, bl in zip(Ps, bufs):
        for k in range(len(P.bufs)):
            if k not in P.out_indices:
                bl[k].write(bl[k].host_ptr, blocking=False)
    for P, bl in zip(Ps, bufs):
        ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, bl), mode="coop", select=1)
    try:
        ctx.finish()
    except Exception as e:
        print("FAIL at step", step, e, flush=True)
        break
    for P, bl in zip(Ps, bufs):
        for k in P.out_indices:
            bl[k].read_array(np.float32)
print("done", step, round(time.time() - t0, 1), ctx.counters(), flush=True)
try:
    ctx.release()
except Exception as e:
    print("release:", e, flush=True)

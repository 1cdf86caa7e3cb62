"""Host time of fcl_enqueue_ndrange (info.t_call_ms, medians over 100 steps) of the bench step's three launches in
GPU-only mode, COOP with selection and COOP without.  Usage: python scripts/t_call.py"""
import os, sys, statistics
sys.path.insert(0, os.environ.get("GRAFT_REPO_ROOT", "/root/repo"))
import fcl_harness as H, workloads as W
from paper_conf_cgo_panditg14_b200 import fcl
ctx = fcl.Context(0)
Ps = [W.make("gesummv", 4096, seed=0, lws1d=256, out_init="zero"), W.make("bicg_s", 4096, 4096, seed=1, lws1d=256, out_init="zero"), W.make("bicg_q", 4096, 4096, seed=2, lws1d=256, out_init="zero")]
bufs = [H.create_buffers(ctx, P) for P in Ps]
res = {}
for mode, sel in (("gpu", 0), ("coop", 1), ("coop", -1)):
    ts = [[] for _ in Ps]
    for r in range(120):
        for q, (P, b) in enumerate(zip(Ps, bufs)):
            info = ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=mode, select=sel)
            ts[q].append(info["t_call_ms"])
        ctx.finish()
    res[f"{mode}{sel}"] = [round(statistics.median(t[20:]) * 1e3, 2) for t in ts]
print(res)

"""Run the bench workload's launches a few times in one mode (for ncu launch lists / captures)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import fcl_harness as H
import workloads as W
from paper_conf_cgo_panditg14_b200 import fcl


def main():
    mode = sys.argv[1] if len(sys.argv) > 1 else "coop"
    reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
    which = sys.argv[3] if len(sys.argv) > 3 else "gesummv_bicg"
    ctx = fcl.Context(0)
    if which == "gesummv_bicg":
        Ps = [W.make("gesummv", 4096, seed=0, lws1d=256, out_init="zero"),
              W.make("bicg_s", 4096, 4096, seed=1, lws1d=256, out_init="zero"),
              W.make("bicg_q", 4096, 4096, seed=2, lws1d=256, out_init="zero")]
    else:
        n = int(which.split(":")[1])
        Ps = [W.make(which.split(":")[0], n, n, seed=0, out_init="zero")]
    launches = []
    for P in Ps:
        bufs = H.create_buffers(ctx, P)
        launches.append(ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, bufs), mode=mode))
    for _ in range(reps):
        for L in launches:
            L()
        ctx.finish()
    print("done", mode, reps, which)


if __name__ == "__main__":
    main()

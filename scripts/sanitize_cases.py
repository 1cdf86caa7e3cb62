"""Small launches of every GPU path for compute-sanitizer (memcheck / racecheck / synccheck):
the persistent dispatcher with the fused merge (free-running, with a slow GPU so that tasks are
skipped and aborted, and forced splits), the plain and lite grids, the diff-merge kernel on raw
buffers, the twin copy, the lazy-return gather, the CORR chain and the upper-triangle GEMMs.
Each result is compared with the GPU-only run bit for bit; prints "sanitize cases ok" at the end.

Streamed inputs are left out: their grid waits, by design, for H2D copies on
another stream, and the sanitizer serialises streams (the 5 s guard would trap).

Usage: compute-sanitizer --tool memcheck python scripts/sanitize_cases.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ.setdefault("FCL_SELECT", "0")
os.environ.setdefault("FCL_NO_STREAM", "1")

import numpy as np

import fcl_harness as H
import workloads as W
from paper_conf_cgo_panditg14_b200 import fcl


def same(a, b, what):
    ua, ub = np.ascontiguousarray(a).view(np.uint32), np.ascontiguousarray(b).view(np.uint32)
    assert np.array_equal(ua, ub), f"{what}: {np.count_nonzero(ua != ub)} words differ"


def main():
    ctx = fcl.Context(0, n_host_threads=4)
    cases = [("gesummv", 256, 256, 32, None), ("atax_y", 200, 300, 32, None), ("syrk", 200, 70, None, (32, 8)),
             ("syr2k", 160, 48, None, (32, 8)), ("conv2d", 150, 300, None, (32, 8)),
             ("corr_reduce", 120, 300, None, (32, 8)), ("corr_corr", 100, 300, 32, None)]
    for kernel, n0, n1, l1, l2 in cases:
        P = W.make(kernel, n0, n1, seed=3, lws1d=l1 or 256, lws2d=l2 or (32, 8))
        ref, _ = H.run(ctx, P, mode="gpu")
        n = P.num_groups
        runs = [dict(forced_split=s) for s in (0, n // 3, n)] + [dict(), dict(gpu_delay_us=200), dict(abort_period=1)]
        for o in runs:
            out, info = H.run(ctx, P, mode="coop", **o)
            for k in P.out_indices:
                same(out[k], ref[k], f"{kernel} {o}")
        out, _ = H.run(ctx, P, mode="cpu")
        for k in P.out_indices:
            same(out[k], ref[k], f"{kernel} cpu")
        print("ok", kernel, flush=True)
    # the dispatcher with the twin captured (Fig 9 as printed) instead of aliased
    os.environ["FCL_FORCE_TWIN"] = "1"
    c2 = fcl.Context(0, n_host_threads=4)
    P = W.make("conv2d", 150, 300, seed=4)
    ref, _ = H.run(c2, P, mode="gpu")
    out, _ = H.run(c2, P, mode="coop", gpu_delay_us=100)
    same(out[1], ref[1], "conv2d twin")
    c2.release()
    # raw diff-merge, all element sizes
    import torch
    for es, dt in ((1, torch.uint8), (2, torch.int16), (4, torch.int32), (8, torch.int64)):
        nb = 1 << 16
        g = torch.randint(0, 100, (nb // es,), device="cuda").to(dt)
        t = torch.randint(0, 100, (nb // es,), device="cuda").to(dt)
        c = t.clone()
        c[::7] += 1
        want = torch.where(c != t, c, g)
        fcl.merge_raw(g.data_ptr(), c.data_ptr(), t.data_ptr(), nb - es, es)   # (a ragged tail)
        torch.cuda.synchronize()
        assert torch.equal(g[:-1], want[:-1]), f"merge es {es}"
    ctx.release()
    print("sanitize cases ok", flush=True)


if __name__ == "__main__":
    main()

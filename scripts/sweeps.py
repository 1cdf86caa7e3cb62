"""SURVEY §8(f) rows 2 and 3 on B200: static-split OracleSP and chunk-sensitivity sweeps
(Figs 2, 3, 13, 17, 18) and the abort / status-location ablation (Fig 15).

  oraclesp : every launch of a config split statically at host fraction f (opts.forced_split:
             the host runs exactly the top f of the work-groups, the GPU is told before it starts);
             OracleSP = the best f.  Reported beside GPU-only, CPU-only and free-running FluidiCL.
  chunks   : free-running FluidiCL with the initial chunk / growth step of C11 swept.
  abort    : in-task poll period (opts.abort_period; -1 = checks at task start only) x status
             word location, for the polling (GEMM-like) kernels: dispatcher time with nothing
             covered and the cooperative step; plus the per-work-group dispatcher overhead
             (T(dispatcher, W = N_wg) - T(plain grid)) / N_wg.

Steps are timed like scripts/bench_configs.py (idle GPU after an L2 flush + read sweep, CUDA
events, all launches of the config + fcl_finish).  One JSON line per point on stdout.
Usage: python scripts/sweeps.py [oraclesp|chunks|abort] ...
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "scripts"))

import torch

import fcl_harness as H
from bench_configs import cfg_problems
from paper_conf_cgo_panditg14_b200 import fcl


class Cfg:
    def __init__(self, name, status="device"):
        self.name = name
        self.Ps, meta = cfg_problems(name)
        self.stream = torch.cuda.Stream()
        self.ctx = fcl.Context(0, status_location=status, streams=(self.stream.cuda_stream, None, None))
        self.bufs = [H.create_buffers(self.ctx, P) for P in self.Ps]
        for dl, db, sl, sb in meta.get("shared", []):
            self.bufs[dl][db] = self.bufs[sl][sb]
        self.reset = meta.get("reset", [])
        self.orig = {li: self.Ps[li].bufs[0].copy() for li in self.reset}
        self.flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
        self.sweep = torch.ones(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")

    def prepared(self, mode, per_launch=None, **kw):
        out = []
        for k, (P, b) in enumerate(zip(self.Ps, self.bufs)):
            o = dict(kw)
            if per_launch:
                o.update(per_launch(k, P))
            out.append(self.ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(self.ctx, P, b), mode=mode, **o))
        return out

    def time(self, launches, reps):
        ts = []
        for r in range(reps + 1):
            for li in self.reset:
                self.bufs[li][0].write_array(self.orig[li])
            self.ctx.finish()
            with torch.cuda.stream(self.stream):
                self.flush.fill_(1.0); self.sweep.sum()
            self.stream.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(self.stream)
            for L in launches:
                L()
            self.ctx.finish()
            e1.record(self.stream)
            e1.synchronize()
            if r >= 1:
                ts.append(e0.elapsed_time(e1))
        return statistics.median(ts)

    def infos(self, launches):
        out = []
        for li in self.reset:
            self.bufs[li][0].write_array(self.orig[li])
        self.ctx.finish()
        for L in launches:
            L()
            self.ctx.finish()
            out.append(self.ctx.launch_info())
        return out

    def release(self):
        seen = set()
        for bl in self.bufs:
            for b in bl:
                if id(b) not in seen:
                    seen.add(id(b))
                    b.release()
        self.ctx.release()


def split_at(frac):
    """forced_split for host fraction `frac` of a launch's work-groups (aligned to WG rows for
    2-D kernels so that the host's share is whole spans)."""
    def f(k, P):
        n = P.num_groups
        unit = (P.gws[0] // P.lws[0]) if len(P.gws) == 2 else 1
        s = n - int(round(frac * n))
        s = max(0, min(n, (s // unit) * unit))
        return {"forced_split": s}
    return f


def oraclesp(names):
    grids = {"atax256": [0, 0.25, 0.5, 0.75, 0.875, 1.0],
             "gesummv_bicg4096": [0, 0.0625, 0.125, 0.25],
             "syrk2048": [0, 0.001, 0.002, 0.005, 0.01],
             "syr2k2048": [0, 0.001, 0.002, 0.005],
             "conv2d16384": [0, 0.1, 0.2, 0.3, 0.4, 0.5, 0.6, 0.8, 1.0],
             "corr4096": [0, 0.001, 0.002, 0.005]}
    for name in names:
        c = Cfg(name)
        reps = 3 if name in ("conv2d16384", "corr4096", "syr2k2048") else 8
        base = {m: c.time(c.prepared(m), reps if m != "cpu" else 1) for m in ("gpu", "coop")}
        base["cpu"] = c.time(c.prepared("cpu"), 1) if name in ("atax256", "gesummv_bicg4096", "conv2d16384") else None
        pts = []
        for f in grids[name]:
            L = c.prepared("coop", per_launch=split_at(f))
            ms = c.time(L, reps)
            pts.append({"host_frac": f, "ms": round(ms, 4)})
            print(json.dumps({"sweep": "oraclesp", "config": name, "host_frac": f, "ms": round(ms, 4)}), flush=True)
        best = min(pts, key=lambda p: p["ms"])
        print(json.dumps({"sweep": "oraclesp_summary", "config": name, "gpu_ms": round(base["gpu"], 4),
                          "cpu_ms": round(base["cpu"], 4) if base["cpu"] else None,
                          "fluidicl_ms": round(base["coop"], 4), "oraclesp_ms": best["ms"],
                          "oraclesp_host_frac": best["host_frac"],
                          "fluidicl_vs_oraclesp": round(best["ms"] / base["coop"], 4)}), flush=True)
        c.release()


def chunks(names):
    for name in names:
        c = Cfg(name)
        reps = 3 if name in ("conv2d16384",) else 8
        for ip in (1, 2, 5, 10, 20):
            for sp in (0, 2, 5):
                L = c.prepared("coop", init_chunk_pct=ip, step_pct=sp)
                ms = c.time(L, reps)
                inf = c.infos(L)
                print(json.dumps({"sweep": "chunks", "config": name, "init_pct": ip, "step_pct": sp, "ms": round(ms, 4),
                                  "cpu_wgs": [i["cpu_wgs"] for i in inf], "n_chunks": [i["n_chunks"] for i in inf]}),
                      flush=True)
        c.release()


def abort(names):
    for name in names:
        for status in ("device", "host_mapped"):
            c = Cfg(name, status=status)
            dom = len(c.Ps) - 1   # the polling launch is the last of every such config
            P = c.Ps[dom]
            plain = c.ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(c.ctx, P, c.bufs[dom]), mode="gpu", timing=True)
            c.infos(c.prepared("gpu"))
            t_plain = statistics.median([c.infos([plain])[0]["t_gpu_kernel_ms"] for _ in range(5)])
            for period in (-1, 1, 4, 8, 32):
                # dispatcher with nothing covered: the host is told it runs [N_wg, N_wg) (W = N_wg)
                disp = c.ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(c.ctx, P, c.bufs[dom]), mode="coop",
                                     timing=True, abort_period=period, forced_split=P.num_groups)
                t_disp = statistics.median([c.infos([disp])[0]["t_gpu_kernel_ms"] for _ in range(5)])
                step = c.time(c.prepared("coop", abort_period=period), 3)
                print(json.dumps({"sweep": "abort", "config": name, "kernel": H.kernel_name(P), "status": status,
                                  "abort_period": period, "plain_kernel_ms": round(t_plain, 4),
                                  "dispatcher_nothing_covered_ms": round(t_disp, 4),
                                  "overhead_per_wg_ns": round((t_disp - t_plain) * 1e6 / P.num_groups, 3),
                                  "coop_step_ms": round(step, 4)}), flush=True)
            c.release()


def main():
    what = sys.argv[1] if len(sys.argv) > 1 else "oraclesp"
    names = sys.argv[2:]
    if what == "oraclesp":
        oraclesp(names or ["atax256", "gesummv_bicg4096", "syrk2048", "conv2d16384", "corr4096"])
    elif what == "chunks":
        chunks(names or ["conv2d16384", "atax256"])
    elif what == "abort":
        abort(names or ["syrk2048", "syr2k2048", "corr4096"])


if __name__ == "__main__":
    main()

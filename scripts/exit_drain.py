"""Exit drain of the persistent dispatcher (SURVEY §8d "Dispatcher"; §6.4 abort in loops,
L20.s44-51, Fig 15 L24.s26-35): the %globaltimer time from the publication of W = 0 (a store
kernel that stamps the clock right after its store, FCL_TEST_PUBLISH_ZERO_US) to the last CTA's
exit from the task loop, in total and divided by the number of CTAs -- for the polling GEMM
bodies at several in-task poll periods (k'-tiles; -1 = checks at task start only) and both
status-word locations.  The host computes nothing in this mode and no merge runs (outputs are
incomplete by construction); one JSON line per point.

Usage: FCL_STATS=1 FCL_TRACE=1 python scripts/exit_drain.py  (the script sets them itself)
"""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CASES = [("syrk", 2048, 2048), ("syr2k", 2048, 2048), ("corr_corr", 4096, 4096)]
PERIODS = [1, 4, 8, 32, -1]
PUBLISH_AFTER_US = 150   # (the GEMM tasks run 0.2-1.5 ms: W = 0 lands in the middle of them)


def child(kernel, n0, n1, period, status):
    sys.path.insert(0, ROOT)
    import fcl_harness as H
    import workloads as W
    from paper_conf_cgo_panditg14_b200 import fcl
    ctx = fcl.Context(0, status_location=status)
    P = W.make(kernel, n0, n1, seed=1, lws1d=256, out_init="zero")
    bufs = H.create_buffers(ctx, P)
    for _ in range(3):
        info = ctx.enqueue_ndrange(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, bufs), mode="coop",
                                   select=-1, abort_period=period)
        ctx.finish()
    info = ctx.launch_info()
    print(json.dumps({"n_wg": info["n_wg"], "gpu_tasks_total": info["gpu_tasks_total"],
                      "gpu_watermark": info["gpu_watermark"]}))
    ctx.release()


def main():
    if len(sys.argv) > 1 and sys.argv[1] == "child":
        child(sys.argv[2], int(sys.argv[3]), int(sys.argv[4]), int(sys.argv[5]), sys.argv[6])
        return
    for status in ("device", "host_mapped"):
        for kernel, n0, n1 in CASES:
            for period in PERIODS:
                trace = os.path.join(ROOT, "gpurun_out", f"drain_{kernel}_{period}_{status}.txt")
                env = dict(os.environ, FCL_STATS="1", FCL_TRACE="1", FCL_TRACE_FILE=trace,
                           FCL_TEST_PUBLISH_ZERO_US=str(PUBLISH_AFTER_US), FCL_SELECT="0")
                out = subprocess.run([sys.executable, __file__, "child", kernel, str(n0), str(n1), str(period), status],
                                     env=env, capture_output=True, text=True, timeout=600)
                info = json.loads(out.stdout.strip().splitlines()[-1]) if out.returncode == 0 else {"error": out.stderr[-400:]}
                # the trace holds the device stamps of every slot; take the last launch's slot
                recs = [l.split() for l in open(trace)] if os.path.exists(trace) else []
                by = {}
                for t, tag, e in recs:
                    if tag.startswith("gpu_"):
                        by.setdefault(int(e), {})[tag] = float(t)
                rows = [d for d in by.values() if "gpu_publish_ns" in d and "gpu_disp_end_ns" in d and "gpu_disp_start_ns" in d]
                row = max(rows, key=lambda d: d["gpu_disp_start_ns"]) if rows else {}
                line = {"kernel": kernel, "n": n0, "status": status, "abort_period": period,
                        "publish_after_us": PUBLISH_AFTER_US, **info}
                if row:
                    ctas = min(info.get("gpu_tasks_total", 0), 148 * (1 if kernel != "corr_corr" else 2))
                    drain = (row["gpu_disp_end_ns"] - row["gpu_publish_ns"]) * 1e3   # ms -> us
                    line.update({"publish_from_start_us": round((row["gpu_publish_ns"] - row["gpu_disp_start_ns"]) * 1e3, 2),
                                 "exit_drain_us": round(drain, 2), "ctas": ctas,
                                 "exit_drain_per_cta_ns": round(drain * 1e3 / max(1, ctas), 1)})
                print(json.dumps(line), flush=True)


if __name__ == "__main__":
    main()

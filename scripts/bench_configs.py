"""Per-configuration measurements: E2E-kernel step time in COOP / GPU-only /
CPU-only mode, the dominant kernel's CUDA-event time and roofline fraction, cooperative
share statistics.  One JSON line per configuration (written to stdout).

Usage: python scripts/bench_configs.py [config ...]   (default: all)
"""
import gc
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np
import torch

import fcl_harness as H
import workloads as W
from paper_conf_cgo_panditg14_b200 import fcl

HBM = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
# FP32 FFMA peak: 148 SMs x 128 FP32 lanes x 2 flop x 1.965 GHz
FP32_TFLOPS = 148 * 128 * 2 * 1.965e9 / 1e12


def cfg_problems(name):
    if name == "atax256":
        P1 = W.make("atax_tmp", 256, 256, seed=0, lws1d=16, out_init="zero")
        P2 = W.make("atax_y", 256, 256, seed=1, lws1d=16, out_init="zero")
        return [P1, P2], {"shared": [(1, 0, 0, 0), (1, 1, 0, 2)]}   # (dst launch, dst buf, src launch, src buf)
    if name == "gesummv_bicg4096":
        P1 = W.make("gesummv", 4096, seed=0, lws1d=256, out_init="zero")
        P2 = W.make("bicg_s", 4096, 4096, seed=1, lws1d=256, out_init="zero")
        P3 = W.make("bicg_q", 4096, 4096, seed=2, lws1d=256, out_init="zero")
        return [P1, P2, P3], {"shared": [(2, 0, 1, 0)]}
    if name == "syrk2048":
        return [W.make("syrk", 2048, 2048, seed=0)], {}
    if name == "syr2k2048":
        return [W.make("syr2k", 2048, 2048, seed=0)], {}
    if name == "conv2d16384":
        return [W.make("conv2d", 16384, 16384, seed=0, out_init="zero")], {}
    if name.startswith("corr"):
        n = m = int(name[4:])
        data = W.corr_chain_inputs(n, m, seed=0)
        Ps = []
        for k in ("corr_mean", "corr_std", "corr_reduce", "corr_corr"):
            P = W.make(k, n, m, seed=0, lws1d=256, out_init="zero")
            P.bufs[0] = data
            Ps.append(P)
        # mean -> std(1), reduce(1); std -> reduce(2); data shared by all
        return Ps, {"shared": [(1, 0, 0, 0), (2, 0, 0, 0), (3, 0, 0, 0), (1, 1, 0, 1), (2, 1, 0, 1), (2, 2, 1, 2)],
                    "reset": [0]}
    raise KeyError(name)


def algorithmic(P):
    """(bound, amount per launch, unit): HBM bytes or FP32 flops the kernel must move / do."""
    n0, n1, k = P.n0, P.n1, P.kernel
    f = 4
    if k in ("atax_tmp", "bicg_q"):
        return "hbm", n0 * n1 * f + n1 * f + n0 * f
    if k in ("atax_y", "bicg_s"):
        return "hbm", n0 * n1 * f + n0 * f + n1 * f
    if k == "gesummv":
        return "hbm", 2 * n0 * n0 * f + 3 * n0 * f
    if k == "syrk":
        return "alu", 2 * n0 * n0 * n1
    if k == "syr2k":
        return "alu", 4 * n0 * n0 * n1
    if k == "conv2d":
        return "hbm", 2 * n0 * n1 * f
    if k in ("corr_mean",):
        return "hbm", n0 * n1 * f + n1 * f
    if k in ("corr_std",):
        return "hbm", n0 * n1 * f + 2 * n1 * f
    if k == "corr_reduce":
        return "hbm", 2 * n0 * n1 * f + 2 * n1 * f
    if k == "corr_corr":
        return "alu", n1 * n1 * n0   # upper triangle: M(M-1)/2 dot products of length N, 2 flop each
    raise KeyError(k)


def run_config(name, steps, cpu_steps, modes):
    Ps, meta = cfg_problems(name)
    stream = torch.cuda.Stream()
    H.unpin_caller()   # the runtime lays its threads out over the creating thread's affinity
    ctx = fcl.Context(0, streams=(stream.cuda_stream, None, None))
    H.pin_caller()
    bufsets = [H.create_buffers(ctx, P) for P in Ps]
    for (dl, db, sl, sb) in meta.get("shared", []):
        if bufsets[dl][db] is not bufsets[sl][sb]:
            bufsets[dl][db].release()
            bufsets[dl][db] = bufsets[sl][sb]
    reset = meta.get("reset", [])
    originals = {li: Ps[li].bufs[0].copy() for li in reset}
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    # read sweep after the write flush: L2 ends full of clean, unrelated lines (no dirty
    # write-backs charged to the next kernel)
    sweep = torch.ones(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda")
    # dominant kernel: the one with the most algorithmic work
    dom = max(range(len(Ps)), key=lambda k: algorithmic(Ps[k])[1] / (HBM * 1e9 if algorithmic(Ps[k])[0] == "hbm" else FP32_TFLOPS * 1e12))
    out = {"config": name, "launches": [H.kernel_name(P) for P in Ps], "dominant": H.kernel_name(Ps[dom])}
    # "mode" or "mode:vK" (host body variant K forced; default: online profiling, C26);
    # "coop_always": COOP without device selection
    def parse(spec):
        mode, _, var = spec.partition(":v")
        hv = int(var) if var else -1
        sel = 0
        if mode == "coop_always":
            mode, sel = "coop", -1
        # a forced variant applies to the kernels that have it; the others run their only body
        hvs = [hv if hv < len(ctx.kernel(H.kernel_name(P)).host_variants) else -1 for P in Ps]
        return mode, hvs, sel

    prepared, prepared_t = {}, {}
    for spec in modes:
        mode, hvs, sel = parse(spec)
        # timed steps without CUDA timing events (they would keep consecutive grids from
        # overlapping); the per-launch detail step below times the dominant kernel
        prepared[spec] = [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=mode,
                                      host_variant=hvs[k], select=sel) for k, (P, b) in enumerate(zip(Ps, bufsets))]
        prepared_t[spec] = [ctx.prepare(H.kernel_name(P), P.gws, P.lws, H.make_args(ctx, P, b), mode=mode,
                                        host_variant=hvs[k], select=sel, timing=(k == dom))
                            for k, (P, b) in enumerate(zip(Ps, bufsets))]

    def one_step(spec):
        for li in reset:     # in-place kernels: restore their input (outside the timed region)
            bufsets[li][0].write_array(originals[li])
        ctx.finish()
        with torch.cuda.stream(stream):
            flush.fill_(1.0); sweep.sum()
        stream.synchronize()   # idle GPU at e0: host work cannot hide under the flush
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for L in prepared[spec]:
            L()
        ctx.finish()
        e1.record(stream)
        e1.synchronize()
        return e0.elapsed_time(e1)

    # GPU-side modes interleaved step by step (slow host/PCIe drifts hit every mode alike); the
    # CPU-only leg separately, with fewer steps -- except for ATAX 256, where FluidiCL's steps run
    # on the host alone (sequence selection): there the CPU-only leg is
    # interleaved too, so that both host-alone legs see the same conditions.  (Interleaved with
    # GESUMMV + BICG the CPU-only steps leave outputs stale on the device, which the GPU-only
    # steps after them pay for: 0.107 against 0.059 ms.)
    ts = {spec: [] for spec in modes}
    first = {}
    gc.collect()
    gc.disable()   # no cyclic collection inside the timed steps
    fast = [m for m in modes if parse(m)[0] != "cpu" or name == "atax256"]
    for rep in range(steps + 2):
        for spec in fast:
            t = one_step(spec)
            if rep == 0:
                first[spec] = t
            if rep >= 2:
                ts[spec].append(t)
    for spec in modes:
        if spec in fast:
            continue
        for rep in range(cpu_steps + 1):
            t = one_step(spec)
            if rep == 0:
                first[spec] = t
            else:
                ts[spec].append(t)
    gc.enable()
    for spec in modes:
        mode = parse(spec)[0]
        c0 = ctx.counters()
        # instrumented steps for per-launch detail (the dominant kernel's CUDA-event time is the
        # median over them, each queued behind an L2 flush: device time, not submission latency)
        kms_list = []
        for rep in range(1 if mode == "cpu" else 5):
            for li in reset:
                bufsets[li][0].write_array(originals[li])
            ctx.finish()
            infos = []
            for k, L in enumerate(prepared_t[spec]):
                if k == dom:
                    with torch.cuda.stream(stream):
                        flush.fill_(1.0); sweep.sum()
                L()
                ctx.finish()
                infos.append(ctx.launch_info())
            if infos[dom]["t_gpu_kernel_ms"] > 0:
                kms_list.append(infos[dom]["t_gpu_kernel_ms"])
        v = ts[spec]
        res = {"step_ms_mean": round(statistics.mean(v), 4), "step_ms_median": round(statistics.median(v), 4),
               "steps": len(v), "first_step_ms": round(first[spec], 4)}
        di = infos[dom]
        if mode != "cpu" and kms_list:
            bound, amt = algorithmic(Ps[dom])
            kms = statistics.median(kms_list)
            if bound == "hbm":
                ach = amt / (kms * 1e-3) / 1e9
                res["roofline"] = {"bound": "hbm", "achieved": round(ach, 1), "peak": HBM, "unit": "GB/s",
                                   "frac": round(ach / HBM, 4), "kernel_ms": round(kms, 4)}
            else:
                ach = amt / (kms * 1e-3) / 1e12
                res["roofline"] = {"bound": "alu", "achieved": round(ach, 2), "peak": round(FP32_TFLOPS, 1),
                                   "unit": "TFLOP/s", "frac": round(ach / FP32_TFLOPS, 4), "kernel_ms": round(kms, 4)}
        res["launch_info"] = [{k: i[k] for k in ("gpu_watermark", "published_watermark", "n_wg", "cpu_wgs", "n_chunks",
                                                 "merged", "cpu_did_all", "gpu_launches", "h2d_bytes", "d2h_bytes",
                                                 "chunk_sizes", "host_variant", "profile_ms_per_wg", "gpu_path",
                                                 "selected", "probe")} for i in infos]
        out[spec] = res
    if "gpu" in out and "cpu" in out and "coop" in out:
        g, c, p = out["gpu"]["step_ms_mean"], out["cpu"]["step_ms_mean"], out["coop"]["step_ms_mean"]
        ideal = 1.0 / (1.0 / g + 1.0 / c)
        out["summary"] = {"gpu_ms": g, "cpu_ms": c, "coop_ms": p, "ideal_ms": round(ideal, 4),
                          "coop_vs_best_single": round(min(g, c) / p, 4), "frac_of_ideal": round(ideal / p, 4)}
        if "coop_always" in out:
            a = out["coop_always"]["step_ms_mean"]
            out["summary"].update({"coop_always_ms": a, "coop_always_vs_best_single": round(min(g, c) / a, 4)})
    out["counters"] = ctx.counters()
    done = set()
    for bl in bufsets:
        for b in bl:
            if id(b) not in done:
                done.add(id(b))
                b.release()
    ctx.release()
    return out


def main():
    args = sys.argv[1:]
    modes = ["gpu", "coop", "coop_always", "cpu"]
    if args and args[0].startswith("--modes="):
        modes = args[0].split("=", 1)[1].split(",")
        args = args[1:]
    names = args or ["atax256", "gesummv_bicg4096", "syrk2048", "syr2k2048", "conv2d16384", "corr4096"]
    for name in names:
        steps = 40 if name not in ("conv2d16384", "corr4096") else 20
        cpu_steps = 3 if name in ("conv2d16384", "syrk2048", "syr2k2048") else (1 if name in ("corr4096", "corr1024") else 10)
        t0 = time.time()
        res = run_config(name, steps, cpu_steps, modes)
        res["wall_s"] = round(time.time() - t0, 1)
        print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()

"""Diff-merge microbench (BASELINE config 5): fcl_merge_raw on 1 MiB .. 16 GiB streams with
0 .. 100 % of the words modified (suffix / scatter / runs of 128), u32 elements (and u8/u64 at
one size).  CUDA events on the launching stream, L2 flushed before each repetition for streams
that fit in L2 (< 256 MiB); inputs larger than L2 are streamed from HBM anyway.

Algorithmic bytes per launch: 8 B read per 4-byte word (cpu + twin) + 4 B per changed word.
Prints one JSON line per point; --quick runs a small subset.
"""
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch

from paper_conf_cgo_panditg14_b200 import fcl

PEAK = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
    os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0


def make(nw, frac, structure, dtype=torch.int32, seed=0):
    g = torch.Generator(device="cuda").manual_seed(seed)
    info = torch.iinfo(dtype)
    twin = torch.randint(info.min, info.max, (nw,), dtype=dtype, device="cuda", generator=g)
    gpu = torch.randint(info.min, info.max, (nw,), dtype=dtype, device="cuda", generator=g)
    cpu = twin.clone()
    k = int(round(frac * nw))
    if k:
        if structure == "suffix":
            cpu[nw - k:] ^= 1
        elif structure == "scatter":
            if nw < (1 << 30):
                idx = torch.randperm(nw, device="cuda", generator=g)[:k]
            else:   # too large for a permutation: independent draws (duplicates only lower k)
                idx = torch.randint(0, nw, (k,), device="cuda", generator=g)
            cpu[idx] ^= 1
        else:   # runs of 128 words
            runs = max(1, k // 128)
            nb = max(1, nw // 128)
            starts = (torch.randperm(nb, device="cuda", generator=g)[:runs] if nb < (1 << 30)
                      else torch.randint(0, nb, (runs,), device="cuda", generator=g)) * 128
            idx = (starts[:, None] + torch.arange(128, device="cuda")[None, :]).reshape(-1)
            idx = idx[idx < nw]
            cpu[idx] ^= 1
    return gpu, cpu, twin


def time_merge(gpu, cpu, twin, es, reps=10):
    s = torch.cuda.current_stream()
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device="cuda") if gpu.numel() * es < (256 << 20) else None
    g0 = gpu.clone()
    ts = []
    for r in range(reps + 2):
        gpu.copy_(g0)
        if flush is not None:
            flush.fill_(1.0)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(s)
        fcl.merge_raw(gpu.data_ptr(), cpu.data_ptr(), twin.data_ptr(), gpu.numel() * es, es, s.cuda_stream)
        e1.record(s)
        e1.synchronize()
        if r >= 2:
            ts.append(e0.elapsed_time(e1))
    changed = int((cpu != twin).sum().item())
    return statistics.median(ts), changed


def main():
    quick = "--quick" in sys.argv
    sizes = [1 << 20, 16 << 20, 256 << 20, 1 << 30] if quick else [1 << 20, 16 << 20, 256 << 20, 1 << 30, 4 << 30, 16 << 30]
    fracs = [0.0, 0.1, 1.0] if quick else [0.0, 1e-3, 1e-2, 0.1, 0.5, 1.0]
    structures = ["suffix", "scatter"] if quick else ["suffix", "scatter", "runs"]
    for nbytes in sizes:
        nw = nbytes // 4
        for structure in structures:
            for frac in fracs:
                if structure != "suffix" and frac in (0.0, 1.0):
                    continue
                gpu, cpu, twin = make(nw, frac, structure)
                ms, changed = time_merge(gpu, cpu, twin, 4, reps=10 if nbytes <= (1 << 30) else 4)
                alg = nw * 8 + changed * 4
                gbs = alg / (ms * 1e-3) / 1e9
                print(json.dumps({"bytes_per_stream": nbytes, "elem_size": 4, "structure": structure, "frac": frac,
                                  "ms": round(ms, 4), "alg_bytes": alg, "gbs": round(gbs, 1),
                                  "frac_of_peak": round(gbs / PEAK, 4)}), flush=True)
                del gpu, cpu, twin
                torch.cuda.empty_cache()
    for es, dt in ((1, torch.uint8), (8, torch.int64)):
        nbytes = 1 << 30
        n = nbytes // es
        gpu, cpu, twin = make(n, 0.1, "scatter", dtype=dt if dt != torch.uint8 else torch.int16)
        if es == 1:
            gpu, cpu, twin = gpu.view(torch.uint8)[:nbytes], cpu.view(torch.uint8)[:nbytes], twin.view(torch.uint8)[:nbytes]
        ms, changed = time_merge(gpu, cpu, twin, es, reps=6)
        alg = nbytes * 2 + changed * es
        gbs = alg / (ms * 1e-3) / 1e9
        print(json.dumps({"bytes_per_stream": nbytes, "elem_size": es, "structure": "scatter", "frac": 0.1,
                          "ms": round(ms, 4), "alg_bytes": alg, "gbs": round(gbs, 1),
                          "frac_of_peak": round(gbs / PEAK, 4)}), flush=True)


if __name__ == "__main__":
    main()

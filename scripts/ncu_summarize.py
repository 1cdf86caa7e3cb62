"""Summarise ncu reports of a round into profiles/<tag>_ncu_summary.md and profiles/ncu_traffic.json."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
TAG = sys.argv[1] if len(sys.argv) > 1 else "r01"
SRC = os.environ.get("NCU_SRC", os.path.join(ROOT, "gpurun_out"))
OUT = os.path.join(ROOT, "profiles")
METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_%peak"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm_%peak"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved_occ_%"),
    ("launch__registers_per_thread", "regs"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "fma_pipe_%"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "lsu_%"),
    ("smsp__average_warp_latency_issue_stalled_long_scoreboard", "stall_long_sb"),
]


def raw(rep):
    if rep.endswith(".csv"):   # a raw page exported on the GPU box (ncu -i ... --page raw --csv)
        out = open(rep).read()
    else:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return []
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for m, short in METRICS:
            if m in hdr:
                v = r[hdr.index(m)]
                d[short] = v + ("" if units[hdr.index(m)] in ("", "%") else " " + units[hdr.index(m)])
                d[short + "_raw"] = v
        res.append(d)
    return res


def to_bytes(v, unit_str):
    v = float(v.replace(",", ""))
    u = unit_str.split()[-1] if " " in unit_str else ""
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)


lines = [f"# ncu summary, round {TAG[1:]}", "",
         "Captured under gpurun with `scripts/ncu_round.sh` (`ncu --set full --clock-control none`, one GPU).",
         "Absolute ncu durations are serialised/cold-cache; compare with the CUDA-event numbers in",
         "`profiles/" + TAG + "_configs.jsonl` and the bench line for live timing.", ""]
traffic = {}
for name, rep in [("gesummv, cooperative launch (lite plain grid when single-wave)", "gesummv_coop"), ("gesummv plain grid (GPU-only)", "gesummv_plain"),
                  ("merge_kernel 1 GiB, 10 % changed, suffix (the bench's case)", "merge_suffix10"),
                  ("merge_kernel 1 GiB, 10 % changed, Bernoulli scatter", "merge_scatter10"),
                  ("merge_kernel 1 GiB, 50 % changed, Bernoulli scatter", "merge_scatter50"),
                  ("SYRK 2048 dispatcher", "syrk"), ("SYR2K 2048 dispatcher", "syr2k"),
                  ("SYRK 2048 plain grid (GPU-only; upper-triangle tiles + mirrors)", "syrk_plain"),
                  ("SYR2K 2048 plain grid (GPU-only)", "syr2k_plain"),
                  ("CORR symmat 4096 plain grid (GPU-only; cp.async pipeline)", "corr_plain"),
                  ("2DCONV 16384^2 dispatcher", "conv2d")]:
    p = os.path.join(SRC, f"{TAG}_{rep}.ncu-rep")
    if not os.path.exists(p):
        p = os.path.join(ROOT, "gpurun_out", f"{TAG}_{rep}_raw.csv")
    if not os.path.exists(p):
        continue
    rows = raw(p)
    lines.append(f"## {name}  (`{TAG}_{rep}.ncu-rep`)")
    lines.append("")
    for d in rows:
        lines.append(f"- kernel: `{d['kernel'][:140]}`")
        for m, short in METRICS:
            if short in d:
                lines.append(f"  - {short}: {d[short]}")
        if "dram_read" in d and "dram_write" in d:
            tb = to_bytes(d["dram_read_raw"], d["dram_read"]) + to_bytes(d["dram_write_raw"], d["dram_write"])
            key = {"gesummv_coop": "gesummv", "merge_suffix10": "merge_kernel", "syrk": "syrk", "conv2d": "conv2d",
                   "gesummv_plain": "gesummv_plain", "syrk_plain": "syrk_plain", "syr2k_plain": "syr2k_plain",
                   "corr_plain": "corr_plain", "syr2k": "syr2k", "merge_scatter10": "merge_scatter10",
                   "merge_scatter50": "merge_scatter50"}[rep]
            traffic[key] = int(tb)
            if rep.startswith("merge_") and "duration_raw" in d:
                # algorithmic bytes: 8 B read per 4-byte word (cpu + twin) + 4 B per changed word
                frac = {"merge_suffix10": 0.1, "merge_scatter10": 0.1, "merge_scatter50": 0.5}[rep]
                nw = (1 << 30) // 4
                alg = nw * 8 + frac * nw * 4
                dur = float(d["duration_raw"].replace(",", "")) * {"nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3,
                                                                    "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1.0}.get(
                    d["duration"].split()[-1], 1e-9)
                peak = json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"] if os.path.exists(
                    os.path.join(ROOT, "MEASURED_PEAKS.json")) else 6650.0
                lines.append(f"  - algorithmic: {alg / dur / 1e9:.0f} GB/s = {alg / dur / 1e9 / peak:.3f} of measured HBM "
                             f"({peak:.0f} GB/s); DRAM bytes: {tb / dur / 1e9:.0f} GB/s = {tb / dur / 1e9 / peak:.3f}; "
                             f"DRAM/algorithmic bytes {tb / alg:.3f}")
            lines.append(f"  - dram traffic (read+write): {tb / 1e6:.1f} MB")
    lines.append("")
# launch list shares
lp = os.path.join(ROOT, "gpurun_out", f"{TAG}_launches.csv")
if os.path.exists(lp):
    rows = list(csv.reader(open(lp)))
    hdr = None
    tot, by = 0.0, {}
    for r in rows:
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d["Metric Name"] != "gpu__time_duration.sum":
                continue
            try:
                v = float(d["Metric Value"].replace(",", ""))
            except ValueError:
                continue
            if v != v:   # (nan: a launch ncu could not time)
                continue
            k = d["Kernel Name"].split("(")[0][:80]
            by[k] = by.get(k, 0.0) + v
            tot += v
    lines.append(f"## Launch list of `python bench.py --steps 2 --warmup 3` (`{TAG}_launches.csv`)")
    lines.append("")
    lines.append("| kernel | total ns | share |")
    lines.append("|---|---|---|")
    for k, v in sorted(by.items(), key=lambda kv: -kv[1]):
        lines.append(f"| `{k}` | {v:.0f} | {v / tot:.3f} |")
    lines.append("")
os.makedirs(OUT, exist_ok=True)
open(os.path.join(OUT, f"{TAG}_ncu_summary.md"), "w").write("\n".join(lines) + "\n")
if traffic:   # (never overwrite the committed table with nothing)
    json.dump(traffic, open(os.path.join(OUT, "ncu_traffic.json"), "w"), indent=1)
print("\n".join(lines))
print(traffic)

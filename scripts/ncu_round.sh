#!/bin/bash
# ncu evidence for one round (run under gpurun; one GPU).  Writes gpurun_out/<tag>_*.
set -x
TAG=${1:-r01}
SKIP_BENCH=${2:-0}
mkdir -p gpurun_out
# reports go to a scratch directory on the box (gpurun brings back at most 64 MiB); the summary,
# per-report raw CSVs and the launch list are written to gpurun_out/ at the end
R=${NCU_DIR:-/tmp/ncu_${TAG}}
mkdir -p $R
# launch list of the bench command itself (cold-cache, serialised: compare shares, not absolutes)
if [ "$SKIP_BENCH" = "0" ]; then
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
    python bench.py --steps 2 --warmup 3 > gpurun_out/${TAG}_bench_under_ncu.log 2>&1
fi
# the dominant kernel of the bench (GESUMMV, cooperative launch: the lite plain grid when it
# runs in one wave, else the dispatcher) and its GPU-only plain grid, full sets
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:.*_kernel.*RowDotBody<float, .*2>' -s 2 -c 1 \
    -o $R/${TAG}_gesummv_coop python scripts/profile_step.py coop 3 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:plain_kernel.*RowDotBody<float, .*2>' -s 2 -c 1 \
    -o $R/${TAG}_gesummv_plain python scripts/profile_step.py gpu 3 > /dev/null 2>&1
# the merge kernel at 1 GiB: the bench's case (10 % suffix) and the worst case (Bernoulli
# scatter, 10 % and 50 % of the words), each capture named after its pattern
for M in "suffix 0.1 suffix10" "scatter 0.1 scatter10" "scatter 0.5 scatter50"; do
    set -- $M
    ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:merge_kernel' -s 2 -c 1 \
        -o $R/${TAG}_merge_$3 python scripts/merge_one.py $1 $2 > /dev/null 2>&1
done
# compute-bound dispatcher: SYRK 2048 and the 2DCONV stencil
FCL_SELECT=0 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:coop_kernel.*GemmBody<float, (\(int\))?0' -s 1 -c 1 \
    -o $R/${TAG}_syrk python scripts/profile_step.py coop 2 syrk:2048 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:plain_kernel.*GemmBody<float, (\(int\))?0' -s 1 -c 1 \
    -o $R/${TAG}_syrk_plain python scripts/profile_step.py gpu 2 syrk:2048 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:plain_kernel.*GemmBody<float, (\(int\))?1' -s 1 -c 1 \
    -o $R/${TAG}_syr2k_plain python scripts/profile_step.py gpu 2 syr2k:2048 > /dev/null 2>&1
FCL_SELECT=0 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:coop_kernel.*GemmBody<float, (\(int\))?1' -s 1 -c 1 \
    -o $R/${TAG}_syr2k python scripts/profile_step.py coop 2 syr2k:2048 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:plain_kernel.*GemmBody<float, (\(int\))?2' -s 1 -c 1 \
    -o $R/${TAG}_corr_plain python scripts/profile_step.py gpu 2 corr_corr:4096 > /dev/null 2>&1
FCL_SELECT=0 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:coop_kernel.*Conv2DBody<float>' -s 1 -c 1 \
    -o $R/${TAG}_conv2d python scripts/profile_step.py coop 2 conv2d:16384 > /dev/null 2>&1
for f in $R/*.ncu-rep; do ncu -i $f --page raw --csv > gpurun_out/$(basename $f .ncu-rep)_raw.csv 2>/dev/null; done
NCU_SRC=$R python scripts/ncu_summarize.py ${TAG}
cp profiles/${TAG}_ncu_summary.md profiles/ncu_traffic.json gpurun_out/ 2>/dev/null
ls -la $R gpurun_out/ | tail -40

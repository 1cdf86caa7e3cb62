#!/bin/bash
# ncu evidence for one round (run under gpurun; one GPU).  Writes gpurun_out/<tag>_*.
set -x
TAG=${1:-r01}
SKIP_BENCH=${2:-0}
mkdir -p gpurun_out
# launch list of the bench command itself (cold-cache, serialised: compare shares, not absolutes)
if [ "$SKIP_BENCH" = "0" ]; then
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
    python bench.py --steps 2 --warmup 3 > gpurun_out/${TAG}_bench_under_ncu.log 2>&1
fi
# the dominant kernel of the bench (GESUMMV, cooperative launch: the lite plain grid when it
# runs in one wave, else the dispatcher) and its GPU-only plain grid, full sets
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:.*_kernel.*RowDotBody<float, .*2>' -s 2 -c 1 \
    -o gpurun_out/${TAG}_gesummv_coop python scripts/profile_step.py coop 3 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:plain_kernel.*RowDotBody<float, .*2>' -s 2 -c 1 \
    -o gpurun_out/${TAG}_gesummv_plain python scripts/profile_step.py gpu 3 > /dev/null 2>&1
# the merge kernel at 1 GiB / 10 % scattered changes
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:merge_kernel' -s 2 -c 1 \
    -o gpurun_out/${TAG}_merge python scripts/merge_one.py > /dev/null 2>&1
# compute-bound dispatcher: SYRK 2048 and the 2DCONV stencil
FCL_SELECT=0 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:coop_kernel.*GemmBody<float, (\(int\))?0' -s 1 -c 1 \
    -o gpurun_out/${TAG}_syrk python scripts/profile_step.py coop 2 syrk:2048 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:plain_kernel.*GemmBody<float, (\(int\))?0' -s 1 -c 1 \
    -o gpurun_out/${TAG}_syrk_plain python scripts/profile_step.py gpu 2 syrk:2048 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:plain_kernel.*GemmBody<float, (\(int\))?1' -s 1 -c 1 \
    -o gpurun_out/${TAG}_syr2k_plain python scripts/profile_step.py gpu 2 syr2k:2048 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:plain_kernel.*GemmBody<float, (\(int\))?2' -s 1 -c 1 \
    -o gpurun_out/${TAG}_corr_plain python scripts/profile_step.py gpu 2 corr_corr:4096 > /dev/null 2>&1
FCL_SELECT=0 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k 'regex:coop_kernel.*Conv2DBody<float>' -s 1 -c 1 \
    -o gpurun_out/${TAG}_conv2d python scripts/profile_step.py coop 2 conv2d:16384 > /dev/null 2>&1
ls -la gpurun_out/

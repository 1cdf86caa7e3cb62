# per-step host trace + GPU stamps (diagnostic; run under gpurun); TRACE_FLUSH=1: bench-like
for m in coop; do
  TRACE_FLUSH=1 FCL_TRACE_FILE=gpurun_out/trace_$m.raw timeout 200 python scripts/trace_step.py $m atax256 > gpurun_out/trace_$m.txt 2>&1
done

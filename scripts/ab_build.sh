#!/bin/bash
# A/B build variants on the GPU box: for each "label|FCL_NVCC_EXTRA" pair, force-rebuild and run
# scripts/bench_configs.py on the configs given in CONFIGS.  Output: gpurun_out/ab_<label>.jsonl
CONFIGS=${CONFIGS:-"syrk2048 syr2k2048 corr4096"}
for v in "$@"; do
  label=${v%%|*}; extra=${v#*|}
  FCL_NVCC_EXTRA="$extra" python paper_conf_cgo_panditg14_b200/_build.py --force > /dev/null 2>&1 || { echo "build $label failed"; continue; }
  python scripts/bench_configs.py $CONFIGS > gpurun_out/ab_${label}.jsonl 2>&1
  python - "$label" <<'PY'
import json, sys
for l in open(f"gpurun_out/ab_{sys.argv[1]}.jsonl"):
    if not l.startswith("{"): continue
    d = json.loads(l)
    print(sys.argv[1], d["config"], "gpu", d["gpu"]["step_ms_median"], d["gpu"].get("roofline", {}).get("kernel_ms"),
          d["gpu"].get("roofline", {}).get("frac"), "coop", d["coop"]["step_ms_median"], d["coop"].get("roofline", {}).get("frac"))
PY
done

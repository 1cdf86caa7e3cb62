# A/B of CORR symmat's cp.async stage shape (k-rows per stage x stages): force-rebuild per variant,
# CUDA-event time of the plain grid at 4096 (scripts/kernel_time.py).  Output: one block per variant.
# Stages above 40 KB go to dynamic shared memory (GemmBody::kDynSmem).
for v in "$@"; do
  label=${v%%|*}; extra=${v#*|}
  FCL_NVCC_EXTRA="$extra" python paper_conf_cgo_panditg14_b200/_build.py --force > /dev/null 2>&1 || { echo "build $label failed"; continue; }
  echo "$label $extra"; python scripts/kernel_time.py corr_corr:4096:4096:256 corr_corr:4096:4096:256
done

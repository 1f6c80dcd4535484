#!/bin/bash
# ncu DRAM bytes of one gate/up launch (layer 0 of the timed region) per group / hints setting
cd $GRAFT_REPO_ROOT
for cfg in "g16h1 BAT_GEMM_GROUP_SWIGLU=16 BAT_GEMM_HINTS=1" "g32h1 BAT_GEMM_GROUP_SWIGLU=32 BAT_GEMM_HINTS=1" "g32h3 BAT_GEMM_GROUP_SWIGLU=32 BAT_GEMM_HINTS=3" "g8h1 BAT_GEMM_GROUP_SWIGLU=8 BAT_GEMM_HINTS=1"; do
  set -- $cfg; tag=$1; shift
  env "$@" BAT_PROFILE_RANGE=1 timeout 600 ncu --profile-from-start off --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum \
    --clock-control none -k regex:gemm2_tc_kernel --launch-skip 2 --launch-count 1 --csv --log-file gpurun_out/swt_$tag.csv \
    python bench.py --steps 1 --warmup 1 --plans 2 --no-cpu-baseline --no-extras --corpus 16384 > /dev/null 2>&1
  python - "$tag" <<'PY'
import csv, sys
tag = sys.argv[1]
rows = [r for r in csv.reader(open(f"gpurun_out/swt_{tag}.csv")) if len(r) > 5]
h = rows[0]
out = {}
for r in rows[1:]:
    out[r[h.index("Metric Name")]] = (r[h.index("Metric Value")], r[h.index("Metric Unit")], r[h.index("Kernel Name")][:30])
print(tag, out)
PY
done

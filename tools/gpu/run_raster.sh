#!/bin/bash
# GEMM rasterisation-group sweep: SwiGLU (1-CTA, 128-row M-tiles) and pair kernels (256-row M-tiles)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
export PYTHONUNBUFFERED=1
timeout 300 python -m pytest tests/test_gpu_kernels.py -q -x -p no:cacheprovider -k gemm > gpurun_out/rs_tests.log 2>&1
echo "gemm tests exit $?"; tail -1 gpurun_out/rs_tests.log
ARGS="--steps 6 --warmup 3 --no-cpu-baseline"
for rep in 1 2; do
for cfg in "8 8 0" "16 8 0" "32 8 0" "65 8 0" "8 16 0" "8 8 1" "8 8 3" "32 8 1"; do
  set -- $cfg
  BAT_GEMM_HINTS=$3 BAT_GEMM_GROUP_SWIGLU=$1 BAT_GEMM_GROUP_M=$2 timeout 300 python bench.py $ARGS > gpurun_out/rs_$1_$2_$3_$rep.json 2>/dev/null
  python - $1 $2 $3 $rep <<'PY'
import json,sys
a,b,h,r=sys.argv[1:]
try: d=json.loads(open(f"gpurun_out/rs_{a}_{b}_{h}_{r}.json").read().strip().splitlines()[-1])
except Exception as e: print(a,b,r,"fail",e); sys.exit()
k=d['kernels']
print(f"swiglu_g={a} pair_g={b} hints={h} rep={r}: {d['value']:.1f} req/s clk {d['clocks']['sm_mhz']} gate_up {k['gemm_gate_up']['tflops']:.0f} down {k['gemm_down']['tflops']:.0f} qkv {k['gemm_qkv']['tflops']:.0f} o {k['gemm_o']['tflops']:.0f} TF/s")
PY
done; done
for g in 8 32; do for h in 0 1; do
BAT_GEMM_HINTS=$h BAT_GEMM_GROUP_SWIGLU=$g BAT_PROFILE_RANGE=1 timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --profile-from-start off -k regex:"gemm" -c 8 --csv python bench.py --steps 1 --warmup 1 --no-cpu-baseline --plans 1 --corpus 2048 > gpurun_out/rs_ncu_${g}_$h.csv 2>/dev/null
echo "ncu g=$g h=$h exit $?"
grep -E "dram__bytes|gpu__time" gpurun_out/rs_ncu_${g}_$h.csv | awk -F'","' '{print $5, $(NF-2), $NF}' | cut -c1-150
done; done

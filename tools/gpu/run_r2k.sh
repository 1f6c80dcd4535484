#!/bin/bash
# round-2 final-code validation: GPU tests, smoke, default bench (configs[2], 262,144-item corpus, extras,
# oracle baseline), reference arm, ncu launch list + one --set full capture of the hot kernels, and the
# 2-rank N>1 path on the one GPU
cd $GRAFT_REPO_ROOT
export PYTHONUNBUFFERED=1
T=r2k
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/${T}_gpu.txt
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider --durations=10 > gpurun_out/${T}_gputests.log 2>&1
echo "pytest rc=$?" >> gpurun_out/${T}_gputests.log; tail -3 gpurun_out/${T}_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${T}_smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/${T}_smoke.log; tail -2 gpurun_out/${T}_smoke.log
timeout 1800 python bench.py > gpurun_out/${T}_bench.json 2> gpurun_out/${T}_bench.err; echo "bench rc=$?" >> gpurun_out/${T}_bench.err; tail -2 gpurun_out/${T}_bench.err
python tools/bench_line.py $T gpurun_out/${T}_bench.json
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/${T}_ref.json 2> gpurun_out/${T}_ref.err; echo "ref rc=$?"
export BAT_PROFILE_RANGE=1
timeout 1200 ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${T}.csv python bench.py --steps 1 --warmup 1 --plans 2 --no-cpu-baseline --no-extras > gpurun_out/${T}_prof1.log 2>&1
echo "list rc=$?"
timeout 1500 ncu --profile-from-start off --set full --clock-control none --import-source on \
  -k regex:"gemm_tc_kernel|gemm2_tc_kernel|attn_tc_kernel|rmsnorm" -c 7 -o gpurun_out/full_${T} \
  python bench.py --steps 1 --warmup 1 --plans 2 --no-cpu-baseline --no-extras > gpurun_out/${T}_prof2.log 2>&1
echo "full rc=$?"
unset BAT_PROFILE_RANGE
BAT_BENCH_SHARED_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 4 --warmup 3 --corpus 32768 --batch 32 --no-extras --no-cpu-baseline > gpurun_out/${T}_bench2.json 2> gpurun_out/${T}_bench2.err; echo "bench2 rc=$?"

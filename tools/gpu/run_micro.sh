#!/bin/bash
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for t in mma_rate mma_contention mma_smem; do echo "== $t"; timeout 120 ./tools/$t 2>&1 | tail -20; done > gpurun_out/micro.txt 2>&1
cat gpurun_out/micro.txt

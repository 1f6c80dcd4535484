#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 120 ./tools/fa4_chain > gpurun_out/fa4_chain.txt 2>&1
cat gpurun_out/fa4_chain.txt

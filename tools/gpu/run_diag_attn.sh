#!/bin/bash
cd $GRAFT_REPO_ROOT
timeout 900 python tools/diag_attn_fullbatch.py 64 2.0 > gpurun_out/diag_attn.log 2>&1
timeout 600 python tools/diag_attn_fullbatch.py 4 2.0 > gpurun_out/diag_attn4.log 2>&1
tail -5 gpurun_out/diag_attn.log

#!/bin/bash
# validation of the current default path + its ncu launch list / full capture, one box call
TAG=${1:-val}
cd $GRAFT_REPO_ROOT
bash tools/gpu/run_final.sh $TAG
bash tools/gpu/run_prof_final.sh $TAG

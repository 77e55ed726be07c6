#!/bin/bash
# round-2 batch 2: full GPU suite on the pruned library, then the ncu counter captures (C2, C5)
cd $GRAFT_REPO_ROOT
python -m pytest tests -m gpu -x -q --durations=8 2>&1 | tail -14 > gpurun_out/b2_pytest.txt
NLAUNCH=80 bash scripts/gpu_prof_r2.sh C2 gpurun_out/prof_r2_C2
NLAUNCH=80 bash scripts/gpu_prof_r2.sh C5 gpurun_out/prof_r2_C5
cat gpurun_out/b2_pytest.txt

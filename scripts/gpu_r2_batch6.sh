#!/bin/bash
# round-2 batch 6: full GPU suite (sector-aligned runs), Fig. 11 / 14 sweeps on C3, slice study on C5
cd $GRAFT_REPO_ROOT
python -m pytest tests -m gpu -x -q --durations=10 2>&1 | tail -16 > gpurun_out/b6_pytest.txt
python scripts/sweep_fig11.py C3 --reps 2 > gpurun_out/r2_fig11_C3.jsonl 2> gpurun_out/fig11.err
python scripts/slice_study.py C5 --reps 2 > gpurun_out/slices_C5.jsonl 2> gpurun_out/slices.err
cat gpurun_out/b6_pytest.txt

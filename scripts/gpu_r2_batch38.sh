#!/bin/bash
# round-2 batch 38: C5 slice study (1 / 2 / 4 / 8 row blocks, every rank alone on the GPU) at the final code
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python scripts/slice_study.py C5 --reps 2 > gpurun_out/b38_slices_C5.jsonl 2> gpurun_out/b38_slices.err
cut -c1-160 gpurun_out/b38_slices_C5.jsonl

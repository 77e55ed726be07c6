#!/bin/bash
# round-2 batch 39: ncu --set full source capture of the final B-Limited merge kernel on C5 (one launch)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 700 ncu --set full --clock-control none --import-source on -k "regex:k_merge_limited" -c 1 \
    -o gpurun_out/prof_b39_C5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_b39.log 2>&1
echo "ncu exit $?"

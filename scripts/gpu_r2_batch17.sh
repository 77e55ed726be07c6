#!/bin/bash
# round-2 batch 17 (evidence at HEAD): DRAM / L2 / atomic / instruction counters of one C5 and one C3
# step (profiles/r2_traffic_*.json), ncu --set full source captures of the top C5 kernels, launch list
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
NLAUNCH=120 bash scripts/gpu_prof_r2.sh C5 gpurun_out/prof_b17_C5
NLAUNCH=120 bash scripts/gpu_prof_r2.sh C3 gpurun_out/prof_b17_C3
timeout 1500 ncu --set full --clock-control none --import-source on -k "regex:k_merge_limited|k_compact_flat|k_expand_blocks" -c 3 \
    -o gpurun_out/prof_b17_full_C5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_b17_full.log 2>&1
echo "ncu full exit $?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/b17_launches_C5.csv \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_b17_launch.log 2>&1
echo "launch list exit $?"

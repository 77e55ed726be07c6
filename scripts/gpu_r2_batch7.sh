#!/bin/bash
# round-2 batch 7: baseline bench line at HEAD (C5 default), then ncu source captures of the
# B-Limited merge and the 4K bucket bin on C5 (instructions per source line)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b7_bench_C5.jsonl 2> gpurun_out/b7_bench.err
tail -1 gpurun_out/b7_bench_C5.jsonl
timeout 1500 ncu --set full --clock-control none --import-source on -k "regex:k_merge_limited|k_merge_bucket<8" -s 0 -c 2 \
    -o gpurun_out/prof_b7_C5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_b7.log 2>&1
echo "ncu exit $?"; tail -2 gpurun_out/ncu_b7.log

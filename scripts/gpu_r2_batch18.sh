#!/bin/bash
# round-2 batch 18: warp-per-row bucket sort for rows of <= 256 slots (reserved[11] = 1) vs the warp
# merge path (+ the per-tile unit map of the flat expansion): parity cases, then C4 / C2 / C5 lines both ways
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "C1 or random_tiny or computed" 2>&1 | tail -3 > gpurun_out/b18_pytest.txt
cat gpurun_out/b18_pytest.txt
for cfg in C4 C2 C5; do
  timeout 400 python bench.py --config $cfg --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b18_bench_${cfg}_wmp.jsonl 2> gpurun_out/b18_${cfg}.err
  python scripts/bench_show.py gpurun_out/b18_bench_${cfg}_wmp.jsonl | tail -2
  SPGEMM_RESERVED=11=1 timeout 400 python bench.py --config $cfg --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b18_bench_${cfg}_wb.jsonl 2>> gpurun_out/b18_${cfg}.err
  python scripts/bench_show.py gpurun_out/b18_bench_${cfg}_wb.jsonl | tail -2
done
timeout 420 ncu --set full --clock-control none --import-source on -k "regex:k_expand_flat|k_merge_wmp" -c 2 \
    -o gpurun_out/prof_b18_C4 python bench.py --config C4 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_b18.log 2>&1
echo "ncu exit $?"

#!/bin/bash
# round-2 batch 13: one-level long-row merge (k_merge_long1) -- parity subset, then C5 / C3 / C2 lines
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "limited or clustered or c_matches or random_tiny or computed or stage2" 2>&1 | tail -4 > gpurun_out/b13_pytest.txt
cat gpurun_out/b13_pytest.txt
for cfg in C5 C3 C2; do
  timeout 900 python bench.py --config $cfg --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b13_bench_$cfg.jsonl 2> gpurun_out/b13_$cfg.err
  python scripts/bench_show.py gpurun_out/b13_bench_$cfg.jsonl | tail -2
done

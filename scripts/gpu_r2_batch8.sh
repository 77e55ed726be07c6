#!/bin/bash
# round-2 batch 8: micro-block expansion of the gathered Low performers + B-Limiting 1/2/4 limited
# blocks per SM (k_merge_limited<NT>): limited-path tests, then C5 / C3 / C2 bench lines per setting
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "limited or expansion or stage3 or c_matches" 2>&1 | tail -4 > gpurun_out/b8_pytest.txt
cat gpurun_out/b8_pytest.txt
for cfg in C5 C3; do
  for lim in 1 2 4; do
    timeout 900 python bench.py --config $cfg --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --opt limit_ctas_per_sm=$lim \
      >> gpurun_out/b8_bench_$cfg.jsonl 2>> gpurun_out/b8_bench.err
    python scripts/bench_show.py gpurun_out/b8_bench_$cfg.jsonl | tail -2
  done
done
timeout 600 python bench.py --config C2 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b8_bench_C2.jsonl 2>> gpurun_out/b8_bench.err
python scripts/bench_show.py gpurun_out/b8_bench_C2.jsonl | tail -2

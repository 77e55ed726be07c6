#!/bin/bash
# round-2 batch 15: B-Limited column groups sorted by two 512-thread sub-groups side by side;
# capped small-block scratch.  Limited tests, then C5 / C3 lines (default and reserved[10] = 1)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "limited or clustered or c_matches or computed" 2>&1 | tail -4 > gpurun_out/b15_pytest.txt
cat gpurun_out/b15_pytest.txt
for cfg in C5 C3; do
  SPGEMM_RESERVED=1=3 timeout 900 python bench.py --config $cfg --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b15_bench_$cfg.jsonl 2> gpurun_out/b15_$cfg.err
  grep unit-profile gpurun_out/b15_$cfg.err | tail -1
  python scripts/bench_show.py gpurun_out/b15_bench_$cfg.jsonl | tail -2
done

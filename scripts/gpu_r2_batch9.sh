#!/bin/bash
# round-2 batch 9: B-Limited per-path clocks (reserved[1] = 3) on C5 at 1 and 2 limited blocks per SM
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for lim in 1 2; do
  SPGEMM_RESERVED=1=3 timeout 900 python bench.py --config C5 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --opt limit_ctas_per_sm=$lim \
     > gpurun_out/b9_C5_$lim.jsonl 2> gpurun_out/b9_C5_$lim.err
  grep unit-profile gpurun_out/b9_C5_$lim.err | tail -1
  python scripts/bench_show.py gpurun_out/b9_C5_$lim.jsonl | tail -1
done

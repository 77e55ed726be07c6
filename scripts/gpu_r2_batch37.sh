#!/bin/bash
# round-2 batch 37: the rest of the GPU suite at HEAD (overflow regression both sides, whole-matrix C4 /
# AB17 / AB18 / C5 in chunks, C3 stage arrays, two ranks on one GPU), C3 / C4 lines
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 300 python -m pytest tests/test_gpu_parity.py -x -q -k "overflow" 2>&1 | tail -1
timeout 1200 python -m pytest tests/test_gpu_full.py tests/test_gpu_dist.py -x -q -k "not C3-opts3 and not C3-opts4 and not C2-opts0 and not C2-opts1 and not C5-opts5" 2>&1 | tail -1
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
for cfg in C3 C4; do
  timeout 300 python bench.py --config $cfg --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b37_bench_$cfg.jsonl 2>> gpurun_out/b37_bench.err
  python scripts/bench_show.py gpurun_out/b37_bench_$cfg.jsonl | tail -2 | head -1
done

#!/bin/bash
# round-2 batch 10: B-Limiting 1 / 2 / 4 per SM with deferral of the heaviest rows; tests; C5 / C3
# lines; ncu source capture of the regular bucket bins (one step of C2)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "limited or clustered" 2>&1 | tail -4 > gpurun_out/b10_pytest.txt
cat gpurun_out/b10_pytest.txt
for cfg in C5 C3; do
  for lim in 1 2 4; do
    SPGEMM_RESERVED=1=3 timeout 900 python bench.py --config $cfg --steps 2 --warmup 2 --no-e2e --no-cpu-baseline --opt limit_ctas_per_sm=$lim \
      >> gpurun_out/b10_bench_$cfg.jsonl 2> gpurun_out/b10_$cfg_$lim.err
    grep unit-profile gpurun_out/b10_$cfg_$lim.err | tail -1
    python scripts/bench_show.py gpurun_out/b10_bench_$cfg.jsonl | tail -2
  done
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_merge_bucket -c 4 \
    -o gpurun_out/prof_b10_C2 python bench.py --config C2 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_b10.log 2>&1
echo "ncu exit $?"

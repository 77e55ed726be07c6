#!/bin/bash
# round-2 batch 34 (final validation at HEAD, after the A/B knob commits): full GPU suite, smoke, default bench line (C5, e2e +
# cpu_baseline), C3 / C2 / C4 lines, ncu launch list of one C5 step
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1300 python -m pytest tests -m gpu -x -q --durations=4 2>&1 | tail -8 > gpurun_out/b34_pytest.txt
cat gpurun_out/b34_pytest.txt
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/b34_smoke.txt 2>&1; tail -1 gpurun_out/b34_smoke.txt
timeout 600 python bench.py > gpurun_out/b34_bench_C5_default.jsonl 2> gpurun_out/b34_bench.err
python scripts/bench_show.py gpurun_out/b34_bench_C5_default.jsonl | tail -2
for cfg in C3 C2 C4; do
  timeout 300 python bench.py --config $cfg --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b34_bench_$cfg.jsonl 2>> gpurun_out/b34_bench.err
  python scripts/bench_show.py gpurun_out/b34_bench_$cfg.jsonl | tail -2
done
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/b34_launches_C5.csv \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/b34_ncu_launch.log 2>&1
echo "launch list exit $?"

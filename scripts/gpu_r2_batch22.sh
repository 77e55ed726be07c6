#!/bin/bash
# round-2 batch 22 (final validation at HEAD): full GPU suite, smoke, default bench line (C5, e2e +
# cpu_baseline), ncu launch list of one step, C5 slice study (1 / 2 / 4 / 8 row blocks)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1300 python -m pytest tests -m gpu -x -q --durations=6 2>&1 | tail -12 > gpurun_out/b22_pytest.txt
cat gpurun_out/b22_pytest.txt
timeout 200 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/b22_smoke.txt 2>&1; tail -2 gpurun_out/b22_smoke.txt
timeout 600 python bench.py > gpurun_out/b22_bench_C5_default.jsonl 2> gpurun_out/b22_bench.err
python scripts/bench_show.py gpurun_out/b22_bench_C5_default.jsonl | tail -2
timeout 400 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/b22_launches_C5.csv \
    python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/b22_ncu_launch.log 2>&1
echo "launch list exit $?"
timeout 600 python scripts/slice_study.py C5 --reps 2 > gpurun_out/b22_slices_C5.jsonl 2> gpurun_out/b22_slices.err
cut -c1-160 gpurun_out/b22_slices_C5.jsonl

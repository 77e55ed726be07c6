#!/bin/bash
# round-2 batch 14: full GPU suite at HEAD, racecheck + memcheck on C1 / tiny / limited paths,
# Fig. 14 B-Limiting sweep (1 / 2 / 4 limited blocks per SM) on C5 and C3, default C5 line
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 1800 python -m pytest tests -m gpu -x -q --durations=8 2>&1 | tail -14 > gpurun_out/b14_pytest.txt
cat gpurun_out/b14_pytest.txt
timeout 900 compute-sanitizer --tool racecheck --print-limit 10 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider \
   -k "c_matches and C1-opts0 or random_tiny and 3 or limited_paths and False-" > gpurun_out/b14_racecheck.log 2>&1
echo "racecheck exit $?" >> gpurun_out/b14_racecheck.log; tail -5 gpurun_out/b14_racecheck.log
timeout 900 compute-sanitizer --tool memcheck --print-limit 10 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider \
   -k "limited or c_matches or random_tiny" > gpurun_out/b14_memcheck.log 2>&1
echo "memcheck exit $?" >> gpurun_out/b14_memcheck.log; tail -4 gpurun_out/b14_memcheck.log
python scripts/sweep_fig11.py C5 --reps 2 --only limit > gpurun_out/b14_fig14_C5.jsonl 2> gpurun_out/b14_fig14.err
python scripts/sweep_fig11.py C3 --reps 2 --only limit > gpurun_out/b14_fig14_C3.jsonl 2>> gpurun_out/b14_fig14.err
cat gpurun_out/b14_fig14_C5.jsonl gpurun_out/b14_fig14_C3.jsonl | cut -c1-220
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/b14_bench_C5_default.jsonl 2> gpurun_out/b14_bench.err
python scripts/bench_show.py gpurun_out/b14_bench_C5_default.jsonl | tail -2

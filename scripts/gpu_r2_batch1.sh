#!/bin/bash
# round-2 batch: parity of the touched paths, C2/C5 lines, C5 slice study, memcheck on C1 / tiny
cd $GRAFT_REPO_ROOT
python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q 2>&1 | tail -3 > gpurun_out/b1_pytest.txt
python bench.py --config C2 --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/b_c2.json 2>&1
python bench.py --config C5 --no-e2e --no-cpu-baseline --steps 3 > gpurun_out/b_c5.json 2>&1
SPGEMM_RESERVED=4=1 python bench.py --config C5 --no-e2e --no-cpu-baseline --steps 3 > gpurun_out/b_c5_r4.json 2>&1
python scripts/slice_study.py C5 --reps 2 > gpurun_out/slices_C5.jsonl 2> gpurun_out/slices.err
timeout 900 compute-sanitizer --tool memcheck --print-limit 10 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "c_matches and (opts0 or opts1 or opts15 or opts19 or opts20) or tiny or limited_paths or window or zeros" > gpurun_out/memcheck.log 2>&1
echo "memcheck exit $?" >> gpurun_out/memcheck.log
cat gpurun_out/b1_pytest.txt; tail -3 gpurun_out/memcheck.log

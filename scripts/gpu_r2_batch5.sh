#!/bin/bash
# round-2 batch 5: GPU suite (minus the whole-matrix full sizes), the 2-rank bench path, smoke, C5 headline line
cd $GRAFT_REPO_ROOT
python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q 2>&1 | tail -3 > gpurun_out/b5_pytest.txt
python -c "import __graft_entry__ as g; g.smoke()" >> gpurun_out/b5_pytest.txt 2>&1
python bench.py > gpurun_out/r2_bench_C5.json 2> gpurun_out/r2_bench_C5.err
cat gpurun_out/b5_pytest.txt; tail -1 gpurun_out/r2_bench_C5.err

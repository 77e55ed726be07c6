#!/bin/bash
# round-2 batch 36: bucket-overflow threshold 127 as default -- parity subset incl. heavy buckets, the
# whole-matrix C3 / C2 / C5 tests, and the default C5 line
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -2 > gpurun_out/b36_pytest_parity.txt; cat gpurun_out/b36_pytest_parity.txt
timeout 1200 python -m pytest tests/test_gpu_full.py -x -q -k "C3 or C2 or C5-opts5" 2>&1 | tail -2 > gpurun_out/b36_pytest_full.txt; cat gpurun_out/b36_pytest_full.txt
timeout 600 python bench.py > gpurun_out/b36_bench_C5_default.jsonl 2> gpurun_out/b36_bench.err
python scripts/bench_show.py gpurun_out/b36_bench_C5_default.jsonl | tail -2

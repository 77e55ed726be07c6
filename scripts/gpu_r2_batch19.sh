#!/bin/bash
# round-2 batch 19: warp bucket sort default for <= 256-slot rows; B-Gathering staging of the tile's A
# values / run bases in the flat expansion.  Parity (C1 / tiny / computed zeros / expansion), then
# C4 / C2 / C5 lines, and C4 with enable_gather = 0 (Fig. 10's B-Gathering switch)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "C1 or random_tiny or computed or expansion or stage3" 2>&1 | tail -3 > gpurun_out/b19_pytest.txt
cat gpurun_out/b19_pytest.txt
for cfg in C4 C2 C5; do
  timeout 400 python bench.py --config $cfg --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b19_bench_${cfg}.jsonl 2> gpurun_out/b19_${cfg}.err
  python scripts/bench_show.py gpurun_out/b19_bench_${cfg}.jsonl | tail -2
done
timeout 400 python bench.py --config C4 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --opt enable_gather=0 > gpurun_out/b19_bench_C4_nogather.jsonl 2>> gpurun_out/b19_C4.err
python scripts/bench_show.py gpurun_out/b19_bench_C4_nogather.jsonl | tail -2
timeout 400 python bench.py --config C2 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --opt enable_gather=0 > gpurun_out/b19_bench_C2_nogather.jsonl 2>> gpurun_out/b19_C2.err
python scripts/bench_show.py gpurun_out/b19_bench_C2_nogather.jsonl | tail -2

#!/bin/bash
# round-2 batch 21: dense-row criterion of the B-Limited kernel (products * d >= span, d = 4 / 2 / 1,
# options.reserved[12]) on C5 / C3 with per-path clocks; C5 slice study at 8 ranks
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
for cfg in C5 C3; do
  for d in 4 2 1; do
    SPGEMM_RESERVED=1=3,12=$d timeout 400 python bench.py --config $cfg --steps 2 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/b21_bench_${cfg}_$d.jsonl 2> gpurun_out/b21_${cfg}_$d.err
    echo "$cfg d=$d"; grep unit-profile gpurun_out/b21_${cfg}_$d.err | tail -1
    python scripts/bench_show.py gpurun_out/b21_bench_${cfg}_$d.jsonl | tail -2
  done
done
timeout 600 python scripts/slice_study.py C5 --reps 2 --parts 8 > gpurun_out/b21_slices_C5_8.jsonl 2> gpurun_out/b21_slices.err
SPGEMM_RESERVED=12=2 timeout 600 python scripts/slice_study.py C5 --reps 2 --parts 8 >> gpurun_out/b21_slices_C5_8.jsonl 2>> gpurun_out/b21_slices.err
cut -c1-300 gpurun_out/b21_slices_C5_8.jsonl

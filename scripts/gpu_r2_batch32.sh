#!/bin/bash
# round-2 batch 32: A/B builds: twice the buckets (LS = 1) in the B-Limited sorts (SPG_LIM_LS) and in the
# 2K / 4K bins (SPG_BIN_LS); parity of both builds, C5 / C3 / C2 lines
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
L=$GRAFT_REPO_ROOT/paper_conf_icde_leekyjkp20_b200
for v in libspgemm_limls libspgemm_binls; do
  SPGEMM_LIB=$L/$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "limited or clustered or C1" 2>&1 | tail -1
done
run() {
  SPGEMM_LIB=$L/$2.so timeout 300 python bench.py --config $1 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b32_$1_$2.jsonl 2> gpurun_out/b32.err
  echo "$1 $2"; python scripts/bench_show.py gpurun_out/b32_$1_$2.jsonl | tail -2
}
for cfg in C5 C3 C2; do run $cfg libspgemm; run $cfg libspgemm_limls; run $cfg libspgemm_binls; done

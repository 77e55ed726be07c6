#!/bin/bash
# round-2 batch 29: A/B builds: software-pipelined B-Limited group sorts (SPG_LIM_GPIPE, C5 / C3) and
# software-pipelined warp-per-row bins (SPG_WB_PIPE, C4 / C2 / C5); parity of both builds
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
L=$GRAFT_REPO_ROOT/paper_conf_icde_leekyjkp20_b200
for v in libspgemm_gpipe libspgemm_wbpipe; do
  SPGEMM_LIB=$L/$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "limited or clustered or C1 or random_tiny" 2>&1 | tail -1
done
run() {
  SPGEMM_LIB=$L/$2.so timeout 300 python bench.py --config $1 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b29_$1_$2.jsonl 2> gpurun_out/b29.err
  echo "$1 $2"; python scripts/bench_show.py gpurun_out/b29_$1_$2.jsonl | tail -2
}
for cfg in C5 C3; do run $cfg libspgemm; run $cfg libspgemm_gpipe; done
for cfg in C4 C2; do run $cfg libspgemm; run $cfg libspgemm_wbpipe; done
run C5 libspgemm_wbpipe

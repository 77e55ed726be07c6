#!/bin/bash
# round-2 batch 35: A/B build: bucket-overflow threshold 127 instead of 64 (SPG_BUCKET_MAX); parity of
# the heavy-bucket tests; C3 / C5 / C2 lines
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
L=$GRAFT_REPO_ROOT/paper_conf_icde_leekyjkp20_b200
SPGEMM_LIB=$L/libspgemm_bmax.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "limited or clustered or C1 or computed" 2>&1 | tail -1
run() {
  SPGEMM_LIB=$L/$2.so timeout 300 python bench.py --config $1 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b35_$1_$2.jsonl 2> gpurun_out/b35.err
  echo "$1 $2"; python scripts/bench_show.py gpurun_out/b35_$1_$2.jsonl | tail -2
}
for cfg in C3 C5 C2; do run $cfg libspgemm; run $cfg libspgemm_bmax; done

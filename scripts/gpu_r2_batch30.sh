#!/bin/bash
# round-2 batch 30: A/B build: k_merge_bucket register budget for 1024 resident threads per SM (no spills)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
L=$GRAFT_REPO_ROOT/paper_conf_icde_leekyjkp20_b200
run() {
  SPGEMM_LIB=$L/$2.so timeout 300 python bench.py --config $1 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b30_$1_$2.jsonl 2> gpurun_out/b30.err
  echo "$1 $2"; python scripts/bench_show.py gpurun_out/b30_$1_$2.jsonl | tail -2
}
for cfg in C5 C2 C4; do run $cfg libspgemm; run $cfg libspgemm_minb4; done

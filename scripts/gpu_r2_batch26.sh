#!/bin/bash
# round-2 batch 26: A/B builds of the merge-bin shapes (SPG_SHAPE 1: 512 / 1K bins with 4 / 8 warps per
# row and 4 slots per thread; 2: software-pipelined 2K / 4K bins) on C5 / C2 / C3
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
L=$GRAFT_REPO_ROOT/paper_conf_icde_leekyjkp20_b200
run() {
  SPGEMM_LIB=$L/$2.so timeout 300 python bench.py --config $1 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b26_$1_$2.jsonl 2> gpurun_out/b26.err
  echo "$1 $2"; python scripts/bench_show.py gpurun_out/b26_$1_$2.jsonl | tail -2
}
for cfg in C5 C2 C3; do run $cfg libspgemm; run $cfg libspgemm_shape1; run $cfg libspgemm_shape2; done

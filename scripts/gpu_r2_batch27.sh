#!/bin/bash
# round-2 batch 27: A/B build SPG_SHAPE 3: software-pipelined 9216-slot limited bin; limited tests on the
# shape-3 build (SPGEMM_LIB) then C5 / C3
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
L=$GRAFT_REPO_ROOT/paper_conf_icde_leekyjkp20_b200
run() {
  SPGEMM_LIB=$L/$2.so timeout 300 python bench.py --config $1 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b27_$1_$2.jsonl 2> gpurun_out/b27.err
  echo "$1 $2"; python scripts/bench_show.py gpurun_out/b27_$1_$2.jsonl | tail -2
}
SPGEMM_LIB=$L/libspgemm_shape3.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "limited or clustered" 2>&1 | tail -2
for cfg in C5 C3; do run $cfg libspgemm; run $cfg libspgemm_shape3; done

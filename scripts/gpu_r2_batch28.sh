#!/bin/bash
# round-2 batch 28: pipelined 9216-slot limited bin as default (limited / clustered / C1 parity);
# A/B build: coarse scatter by per-group ballots (SPG_SCATTER_BALLOT) on C5 / C3 / C2
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "limited or clustered or C1" 2>&1 | tail -2
L=$GRAFT_REPO_ROOT/paper_conf_icde_leekyjkp20_b200
run() {
  SPGEMM_LIB=$L/$2.so timeout 300 python bench.py --config $1 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b28_$1_$2.jsonl 2> gpurun_out/b28.err
  echo "$1 $2"; python scripts/bench_show.py gpurun_out/b28_$1_$2.jsonl | tail -2
}
for cfg in C5 C3 C2; do run $cfg libspgemm; run $cfg libspgemm_ballot; done

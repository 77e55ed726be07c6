#!/bin/bash
# round-2 batch 25: A/B builds: coarse groups up to 7/8 of the sorter (C5 / C3), flat-expansion tile
# of 1024 / 4096 units (C4 / C2 / C5)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
L=$GRAFT_REPO_ROOT/paper_conf_icde_leekyjkp20_b200
run() {
  SPGEMM_LIB=$L/$2.so timeout 300 python bench.py --config $1 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b25_$1_$2.jsonl 2> gpurun_out/b25.err
  echo "$1 $2"; python scripts/bench_show.py gpurun_out/b25_$1_$2.jsonl | tail -2
}
for cfg in C5 C3; do run $cfg libspgemm; run $cfg libspgemm_t78; done
for cfg in C4 C2 C5; do run $cfg libspgemm_tile1k; run $cfg libspgemm_tile4k; done
run C4 libspgemm

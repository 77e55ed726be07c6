#!/bin/bash
# round-2 batch 24: A/B builds: histogram pad word, compaction chunk / block size (via SPGEMM_LIB)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
L=$GRAFT_REPO_ROOT/paper_conf_icde_leekyjkp20_b200
for cfg in C5 C2; do
  for v in libspgemm libspgemm_nohpad libspgemm_cmp16k libspgemm_cmp4k libspgemm_cmp512; do
    SPGEMM_LIB=$L/$v.so timeout 300 python bench.py --config $cfg --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b24_${cfg}_$v.jsonl 2> gpurun_out/b23.err
    echo "$cfg $v"; python scripts/bench_show.py gpurun_out/b24_${cfg}_$v.jsonl | tail -2
  done
done

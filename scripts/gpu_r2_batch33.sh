#!/bin/bash
# round-2 batch 33: A/B builds: L2 prefetch of the flat-expansion tile's A values / run bases
# (SPG_EXP_PREFETCH=1) and of its B' rows too (=2); expansion parity; C4 / C5 / C2 lines
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
L=$GRAFT_REPO_ROOT/paper_conf_icde_leekyjkp20_b200
for v in libspgemm_pref libspgemm_pref2; do
  SPGEMM_LIB=$L/$v.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "C1 or expansion or random_tiny" 2>&1 | tail -1
done
run() {
  SPGEMM_LIB=$L/$2.so timeout 300 python bench.py --config $1 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b33_$1_$2.jsonl 2> gpurun_out/b33.err
  echo "$1 $2"; python -c "
import json; d=json.loads(open('gpurun_out/b33_$1_$2.jsonl').readlines()[-1]); k=d['kernel_ms']; print(d['ms_per_step'], 'expand', k.get('expand'), 'blocks', k.get('expand_blocks'))"
}
for cfg in C4 C5 C2; do run $cfg libspgemm; run $cfg libspgemm_pref; run $cfg libspgemm_pref2; done

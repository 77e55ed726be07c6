# usage: bash scripts/gpu_variants.sh "0 1 2"
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for v in $1; do
  SPGEMM_MERGE_VARIANT=$v timeout 300 python bench.py --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/bench_v$v.log 2>&1
  echo "variant $v:"; python -c "
import json,sys; d=json.loads(open('gpurun_out/bench_v$v.log').read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], {k:v for k,v in d['kernel_ms'].items() if k.startswith('merge')})"
done

# per-rank step time of an N-way row partition, one rank at a time on one GPU (scaling study)
# usage: bash scripts/gpu_slices.sh C2 "8:0 8:7 4:0 2:0"
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for sl in $2; do
  timeout 900 python bench.py --config $1 --slice $sl --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/slice.log 2>&1
  echo "== $sl exit $?"
  grep '^{' gpurun_out/slice.log | python -c "
import json, sys
for ln in sys.stdin:
    d = json.loads(ln); k = d['kernel_ms']
    print(d['ms_per_step'], 'products', d['config']['products'], 'kernels', round(sum(k.values()), 3), 'launches/step', d['gpu_launches'] // d['steps'])
    print('  ', [(n, round(v, 3)) for n, v in list(k.items())[:14]])"
done

# Fig. 10 ablation on B200: each Block Reorganizer technique switched off in turn (bench.py --opt)
# usage: bash scripts/gpu_ablation.sh "C2 C3"
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
: > gpurun_out/ablation.jsonl
for c in $1; do
  for o in "" "--opt enable_split=0" "--opt enable_gather=0" "--opt enable_split=0 --opt enable_gather=0" "--opt beta=10 --opt enable_limit=1" "--opt beta=10 --opt enable_limit=0"; do
    timeout 400 python bench.py --config $c --steps 3 --warmup 2 --no-e2e --no-cpu-baseline $o > gpurun_out/abl.log 2>&1
    echo "== $c [$o] exit $?"
    grep '^{' gpurun_out/abl.log | python -c "
import json, sys
for ln in sys.stdin:
    d = json.loads(ln); d['ablation'] = '$o'
    print(json.dumps(d), file=open('gpurun_out/ablation.jsonl', 'a'))
    k = d['kernel_ms']
    print(d['value'], d['ms_per_step'], 'expand', round(sum(v for n, v in k.items() if n.startswith('expand')), 3),
          'merge', round(sum(v for n, v in k.items() if n.startswith('merge')), 3))"
  done
done

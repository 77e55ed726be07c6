# A/B of bench configs across git worktrees (each built in place): bash scripts/gpu_ab_worktrees.sh "C5 C3" "wt0 ."
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for c in $1; do
for w in $2; do
  (cd $w && timeout 900 python bench.py --config $c --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /tmp/ab.log 2>&1)
  echo "== $c $w"
  grep '^{' /tmp/ab.log | python -c "
import json,sys
for l in sys.stdin:
  d=json.loads(l); k=d['kernel_ms']; print(d['ms_per_step'], [(n,round(v,2)) for n,v in list(k.items())[:5]])"
done; done

# usage: bash scripts/gpu_configs.sh "C3 C4" [steps]
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for c in $1; do
  timeout 900 python bench.py --config $c --steps ${2:-2} --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
  echo "== $c exit $?"; tail -c 1500 gpurun_out/bench_$c.log
done

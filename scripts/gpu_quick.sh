# usage: bash scripts/gpu_quick.sh "<pytest -k expr>" "C2 C3 ..."   (tests subset, then bench per config)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -20 gpurun_out/build.log; exit 1; }
if [ -n "$1" ]; then
  timeout 1800 python -m pytest tests -m gpu -x -q -k "$1" -p no:cacheprovider > gpurun_out/pytest_q.log 2>&1
  echo "pytest exit $?"; tail -3 gpurun_out/pytest_q.log
fi
for c in $2; do
  timeout 900 python bench.py --config $c --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
  echo "== $c exit $?"
  python - "$c" <<'PY'
import json, sys
for ln in open(f"gpurun_out/bench_{sys.argv[1]}.log"):
    if ln.startswith("{"):
        d = json.loads(ln)
        print(d["value"], d["ms_per_step"], list(d["kernel_ms"].items())[:7])
    elif "rror" in ln:
        print(ln.strip())
PY
done

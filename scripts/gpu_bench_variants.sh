# usage: bash scripts/gpu_bench_variants.sh "1=1" "" ...   (SPGEMM_RESERVED settings; "" = default)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for v in "$@"; do
  SPGEMM_RESERVED="$v" timeout 900 python bench.py --config ${CFG:-C2} --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > gpurun_out/bench_v.log 2>&1
  echo "== [$v] exit $?"
  python - <<'PY'
import json
for ln in open("gpurun_out/bench_v.log"):
    if ln.startswith("{"):
        d = json.loads(ln)
        print(d["value"], d["ms_per_step"], d.get("merge_units"), list(d["kernel_ms"].items())[:6])
    elif "Error" in ln or "error" in ln or "unit-profile" in ln:
        print(ln.strip())
PY
done

# usage: bash scripts/gpu_check.sh [pytest-k-expression]
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
if [ -n "$1" ]; then K="-k $1"; else K=""; fi
timeout 2400 python -m pytest tests -m gpu -x -q -rf --timeout 1200 --durations=8 -p no:cacheprovider $K > gpurun_out/pytest_gpu.log 2>&1
echo "pytest exit $?" >> gpurun_out/pytest_gpu.log
timeout 300 python bench.py --steps 5 --warmup 3 > gpurun_out/bench.log 2>&1
echo "bench exit $?" >> gpurun_out/bench.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/ncu_bench.log 2>&1
echo "ncu exit $?" >> gpurun_out/ncu_bench.log
tail -5 gpurun_out/pytest_gpu.log; tail -c 3000 gpurun_out/bench.log

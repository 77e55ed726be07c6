# usage: bash scripts/gpu_sanitize.sh "<pytest -k expr>"
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 compute-sanitizer --tool memcheck --print-limit 10 python -m pytest tests/test_gpu_parity.py -x -q --timeout 600 -p no:cacheprovider -k "$1" > gpurun_out/sanitize.log 2>&1
echo "sanitize exit $?" >> gpurun_out/sanitize.log
tail -30 gpurun_out/sanitize.log

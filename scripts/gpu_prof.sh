# usage: bash scripts/gpu_prof.sh <kernel-regex> <count> <tag> [bench args...]
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
REGEX=$1; CNT=$2; TAG=$3; shift 3
timeout 1500 ncu --set full --clock-control none --import-source on -k "regex:$REGEX" -s 0 -c $CNT \
    -o gpurun_out/prof_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline "$@" > gpurun_out/ncu_$TAG.log 2>&1
echo "ncu exit $?" >> gpurun_out/ncu_$TAG.log
tail -3 gpurun_out/ncu_$TAG.log

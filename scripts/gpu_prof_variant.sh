# usage: bash scripts/gpu_prof_variant.sh <variant> <kernel-regex> <skip> <count> <tag>
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
SPGEMM_MERGE_VARIANT=$1 timeout 1200 ncu --set full --clock-control none --import-source on -k "regex:$2" -s $3 -c $4 \
    -o gpurun_out/prof_$5 python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline > gpurun_out/ncu_$5.log 2>&1
echo "ncu exit $?"; tail -2 gpurun_out/ncu_$5.log

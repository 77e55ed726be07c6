#!/bin/bash
# B-Limited coarse path knobs on C5 / C3: reserved[10] paired half-CTA group sorts, reserved[11] MATCH scatter
cd $GRAFT_REPO_ROOT
for cfg in C5 C3; do
python bench.py --config $cfg --no-e2e --no-cpu-baseline --steps 2 > gpurun_out/k_${cfg}_00.json 2>&1
SPGEMM_RESERVED=11=1 python bench.py --config $cfg --no-e2e --no-cpu-baseline --steps 2 > gpurun_out/k_${cfg}_01.json 2>&1
SPGEMM_RESERVED=10=1 python bench.py --config $cfg --no-e2e --no-cpu-baseline --steps 2 > gpurun_out/k_${cfg}_10.json 2>&1
SPGEMM_RESERVED=10=1,11=1 python bench.py --config $cfg --no-e2e --no-cpu-baseline --steps 2 > gpurun_out/k_${cfg}_11.json 2>&1
done

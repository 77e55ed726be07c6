#!/bin/bash
# One bench step of config $1 under ncu with the counters bench.py / DESIGN.md cite: DRAM bytes,
# L2 bytes + L2 atomic / reduction sectors, shared-memory atomics, occupancy, duration, for every
# launch of the step (one GPU; never a multi-rank command).  Summarise with scripts/ncu_traffic.py.
#   scripts/gpu_prof_r2.sh C5 gpurun_out/prof_r2_C5
cfg=$1; out=$2; shift 2
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum
M=$M,lts__t_sectors_op_atom.sum,lts__t_sectors_op_red.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum
M=$M,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,launch__registers_per_thread
M=$M,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed
ncu --metrics $M --clock-control none -c ${NLAUNCH:-80} -o $out \
    python bench.py --config $cfg --steps 1 --warmup 0 --no-e2e --no-cpu-baseline "$@" > ${out}.log 2>&1
tail -2 ${out}.log

#!/bin/bash
# ncu evidence for slice recovery (run under gpurun): launch lists of the 32x32-region TMM benches and one
# --set full capture of the list-mode (slice task) tmm_tc_kernel.
mkdir -p gpurun_out
B="python bench.py --steps 2 --warmup 1 --overhead-reps 2 --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_tmm8192_r32.csv $B --workload tmm8192_bf16_r32 > gpurun_out/launches_tmm8192_r32.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_tmm16384_r32.csv $B --workload tmm16384_r32_array > gpurun_out/launches_tmm16384_r32.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tmm_tc_kernel -s 1 -c 1 -o gpurun_out/prof_tmm_tc_slices $B --workload tmm8192_bf16_r32 > gpurun_out/prof_tmm_tc_slices.log 2>&1
ls -la gpurun_out

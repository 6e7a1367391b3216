#!/bin/bash
# ncu evidence pass (run under gpurun, one GPU). Outputs land in gpurun_out/.
#   launch lists (every kernel, cold-cache, serialised) of the default bench and the stencil bench,
#   and one `--set full` capture of each hot kernel.
set -x
mkdir -p gpurun_out
B="python bench.py --steps 2 --warmup 1 --overhead-reps 2 --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_tmm8192.csv $B > gpurun_out/launches_tmm8192.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_stencil.csv $B --workload stencil32768 > gpurun_out/launches_stencil.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tmm_tc2_kernel -s 2 -c 1 -o gpurun_out/prof_tmm_tc2 $B > gpurun_out/prof_tmm_tc2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:tmm_tc_kernel -s 1 -c 1 -o gpurun_out/prof_tmm_tc_recover $B > gpurun_out/prof_tmm_tc_recover.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:validate_kernel -s 3 -c 1 -o gpurun_out/prof_validate_tmm $B > gpurun_out/prof_validate_tmm.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:stencil5_ldg_kernel -s 2 -c 1 -o gpurun_out/prof_stencil $B --workload stencil32768 > gpurun_out/prof_stencil.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:validate_kernel -s 3 -c 1 -o gpurun_out/prof_validate_stencil $B --workload stencil32768 > gpurun_out/prof_validate_stencil.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_spmv.csv $B --workload spmv4m > gpurun_out/launches_spmv.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 2 -c 1 -o gpurun_out/prof_spmv $B --workload spmv4m > gpurun_out/prof_spmv.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:validate_kernel -s 3 -c 1 -o gpurun_out/prof_validate_spmv $B --workload spmv4m > gpurun_out/prof_validate_spmv.log 2>&1
ls -la gpurun_out

#!/bin/bash
# Round-2 ncu evidence pass (run under gpurun, one GPU). Outputs land in gpurun_out/r02/.
#   launch lists (every kernel, cold-cache, serialised) of the default bench line (C4 stencil) and of the
#   C2 TMM lines; one `--set full` capture of each hot kernel.
mkdir -p gpurun_out/r02
B="python bench.py --steps 2 --warmup 1 --overhead-reps 2 --no-cpu-baseline"
N="timeout 900 ncu --clock-control none"
F="--set full --import-source on"
$N --metrics gpu__time_duration.sum -c 400 --csv --log-file gpurun_out/r02/launches_stencil.csv $B > gpurun_out/r02/launches_stencil.log 2>&1
$N --metrics gpu__time_duration.sum -c 400 --csv --log-file gpurun_out/r02/launches_tmm8192.csv $B --workload tmm8192_bf16 > gpurun_out/r02/launches_tmm8192.log 2>&1
$N --metrics gpu__time_duration.sum -c 400 --csv --log-file gpurun_out/r02/launches_tmm8192_f32.csv $B --workload tmm8192_f32 > gpurun_out/r02/launches_tmm8192_f32.log 2>&1
$N $F -k regex:stencil5_ldg_kernel -s 2 -c 1 -o gpurun_out/r02/prof_stencil $B > gpurun_out/r02/prof_stencil.log 2>&1
$N $F -k regex:validate_kernel -s 3 -c 1 -o gpurun_out/r02/prof_validate_stencil $B > gpurun_out/r02/prof_validate_stencil.log 2>&1
$N $F -k regex:tmm_tc2_kernel -s 2 -c 1 -o gpurun_out/r02/prof_tmm_tc2 $B --workload tmm8192_bf16 > gpurun_out/r02/prof_tmm_tc2.log 2>&1
$N $F -k regex:tmm_tc_kernel -s 1 -c 1 -o gpurun_out/r02/prof_tmm_tc_recover $B --workload tmm8192_bf16 > gpurun_out/r02/prof_tmm_tc_recover.log 2>&1
$N $F -k regex:validate_kernel -s 3 -c 1 -o gpurun_out/r02/prof_validate_tmm $B --workload tmm8192_bf16 > gpurun_out/r02/prof_validate_tmm.log 2>&1
$N $F -k regex:tmm_tf32x3_kernel -s 2 -c 1 -o gpurun_out/r02/prof_tmm_tf32 $B --workload tmm8192_f32 > gpurun_out/r02/prof_tmm_tf32.log 2>&1
ls -la gpurun_out/r02
# keep the copy-back small (gpurun merges <= 64 MiB): export every capture to CSV (+ the top SASS lines) and drop
# the .ncu-rep files
for r in gpurun_out/r02/*.ncu-rep; do
  b=${r%.ncu-rep}
  ncu -i $r --page raw --csv > $b.raw.csv 2>/dev/null
  ncu -i $r --page details --csv > $b.details.csv 2>/dev/null
  python tools/ncu_sass_top.py $r 30 > $b.sass_top.txt 2>&1
  rm -f $r
done
du -sh gpurun_out

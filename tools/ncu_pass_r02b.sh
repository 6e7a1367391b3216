#!/bin/bash
# Round-2 ncu pass for the 256-row CLC TMM kernel (the C2 / C3 / C5 body since the CLC change): launch list of the
# tmm8192_bf16 bench command and one --set full capture of tmm_tc4_kernel (CSV exports only).
mkdir -p gpurun_out/r02b
B="python bench.py --steps 2 --warmup 1 --overhead-reps 2 --no-cpu-baseline --workload tmm8192_bf16"
timeout 900 ncu --clock-control none --metrics gpu__time_duration.sum -c 400 --csv --log-file gpurun_out/r02b/launches_tmm8192.csv $B > /dev/null 2>&1
timeout 900 ncu --clock-control none --set full --import-source on -k regex:tmm_tc4_kernel -s 2 -c 1 -o gpurun_out/r02b/prof_tmm_tc4 $B > gpurun_out/r02b/prof_tmm_tc4.log 2>&1
for r in gpurun_out/r02b/*.ncu-rep; do b=${r%.ncu-rep}; ncu -i $r --page raw --csv > $b.raw.csv; ncu -i $r --page details --csv > $b.details.csv; python tools/ncu_sass_top.py $r 30 > $b.sass_top.txt 2>&1; rm -f $r; done
ls gpurun_out/r02b

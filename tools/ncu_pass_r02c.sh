#!/bin/bash
# Round-2 final ncu pass for the default bench line (C4 stencil, two-phase protected body, TMA-fed recovery):
# launch list of the bench command + one --set full capture of the protected body, the twin, the list-mode
# recovery and the validate kernel. Outputs in gpurun_out/r02_final/ (CSV only; .ncu-rep dropped).
D=gpurun_out/r02_final
mkdir -p $D
B="python bench.py --steps 2 --warmup 1 --overhead-reps 2 --no-cpu-baseline"
N="timeout 900 ncu --clock-control none"
F="--set full --import-source on --kernel-name-base mangled"
$N --metrics gpu__time_duration.sum -c 400 --csv --log-file $D/launches_stencil.csv $B > $D/launches_stencil.log 2>&1
$N $F -k regex:stencil5_ldg_kernelILj3ELi0ELi1ELi16ELi3E -s 1 -c 1 -o $D/prof_stencil $B > $D/prof_stencil.log 2>&1
$N $F -k regex:stencil5_ldg_kernelILj0E -s 1 -c 1 -o $D/prof_stencil_twin $B > $D/prof_stencil_twin.log 2>&1
$N $F -k regex:stencil5_tma_kernel -s 1 -c 1 -o $D/prof_stencil_recover $B > $D/prof_stencil_recover.log 2>&1
$N $F -k regex:validate_kernel -s 3 -c 1 -o $D/prof_validate_stencil $B > $D/prof_validate_stencil.log 2>&1
for r in $D/*.ncu-rep; do
  b=${r%.ncu-rep}
  ncu -i $r --page raw --csv > $b.raw.csv 2>/dev/null
  ncu -i $r --page details --csv > $b.details.csv 2>/dev/null
  python tools/ncu_sass_top.py $r 30 > $b.sass_top.txt 2>&1
  bash tools/ncu_brief.sh $r > $b.brief.txt 2>&1
  rm -f $r
done
ls -la $D

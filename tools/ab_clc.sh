#!/bin/bash
# A/B of the 256-row TMM kernel's work distribution: static persistent (LP_TC_CLC=0) vs cluster launch control
# (LP_TC_CLC=1), raster groups LP_TC4_GROUP; DRAM/L2 traffic at 32768^3, C5 vs cuBLAS, 8192^3 bench body.
M=gpu__time_duration.sum,dram__bytes_read.sum,l1tex__m_xbar2l1tex_read_bytes.sum,sm__cycles_elapsed.avg.per_second
for clc in 0 1; do for g in 2 4 8; do
  LP_TC_CLC=$clc LP_TC4_GROUP=$g timeout 600 ncu --metrics $M --clock-control none -k regex:tmm_tc python tools/probe/c5_traffic.py 32768 2>&1 | grep -E "dram__|gpu__time|per_second" | tr -s ' ' | sed "s/^/clc=$clc G=$g /"
done; done
for clc in 1 0; do LP_TC_CLC=$clc timeout 900 python tools/c5_vs_cublas.py 65536 2>&1 | tail -4 | sed "s/^/clc=$clc /"; done
for clc in 1 0; do for i in 1 2; do LP_TC_CLC=$clc python bench.py --workload tmm8192_bf16 --steps 5 --overhead-reps 10 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('clc=$clc 8192', d['t_protected_ms'], d['t_unprotected_ms'], d['roofline']['frac'])"; done; done

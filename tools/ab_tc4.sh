#!/bin/bash
# 256-row (tc4, default) vs 128-row (LP_TC_TILE=128) CTA-pair TMM kernel: C5 vs cuBLAS under the power cap,
# DRAM / L2 traffic at 32768^3 for tc4 raster groups 2/4/8, the 128-row kernel for reference.
mkdir -p gpurun_out
python tools/c5_vs_cublas.py 65536 2>&1 | tail -5 | sed 's/^/tc4 /'
LP_TC_TILE=128 python tools/c5_vs_cublas.py 65536 2>&1 | tail -4 | sed 's/^/tc2 /'
M=gpu__time_duration.sum,dram__bytes_read.sum,l1tex__m_xbar2l1tex_read_bytes.sum,sm__cycles_elapsed.avg.per_second
for g in 2 4 8; do
  LP_TC4_GROUP=$g ncu --metrics $M --clock-control none -k regex:tmm_tc python tools/probe/c5_traffic.py 32768 2>&1 | grep -E "dram__|gpu__time|xbar|per_second" | sed "s/^/tc4 G=$g /"
done
LP_TC_TILE=128 ncu --metrics $M --clock-control none -k regex:tmm_tc python tools/probe/c5_traffic.py 32768 2>&1 | grep -E "dram__|gpu__time|xbar|per_second" | sed "s/^/tc2 /"

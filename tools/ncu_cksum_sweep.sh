#!/bin/bash
# ncu metric sweep of the protected body per checksum type vs the unprotected twin (run under gpurun).
mkdir -p gpurun_out
M=gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__inst_executed_pipe_alu.sum,sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__inst_executed.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,sm__cycles_elapsed.avg.per_second
for w in tmm tmmf32 stencil; do
  case $w in tmm) K="tmm_tc[24]_kernel";; tmmf32) K=tmm_tf32x3_kernel;; stencil) K=stencil5_ldg_kernel;; esac
  timeout 900 ncu --metrics $M --clock-control none -k regex:$K --csv --log-file gpurun_out/cksum_sweep_$w.csv \
    python tools/cksum_sweep_kernels.py --workload $w > gpurun_out/cksum_sweep_$w.log 2>&1
done
ls -la gpurun_out/cksum_sweep_*

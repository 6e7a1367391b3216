#!/bin/bash
# ncu: atomic traffic and time of the protected C3 body per checksum store (order: array, quad_cas, cuckoo, quad_lock)
M=gpu__time_duration.sum,l1tex__t_bytes_pipe_lsu_mem_global_op_atom.sum,l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum,lts__t_sectors_srcunit_tex_op_atom.sum,l1tex__t_bytes_pipe_lsu_mem_global_op_red.sum,dram__bytes_write.sum
for r in 128 32; do
  timeout 1200 ncu --metrics $M --clock-control none -k regex:tmm_tc --csv python tools/store_kernels.py --region $r > gpurun_out/store_atoms_r$r.csv 2> gpurun_out/store_atoms_r$r.err
done

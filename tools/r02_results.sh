#!/bin/bash
# Round-2 results: every bench workload once + the design-space grids (run under gpurun, one GPU).
bash tools/run_results.sh stencil32768 stencil32768_adler tmm8192_bf16 tmm8192_bf16_mod tmm8192_bf16_xor \
  tmm8192_bf16_adler tmm8192_bf16_all tmm8192_bf16_r32 tmm8192_bf16_f32out tmm8192_f32 tmm8192_f32_simt \
  tmm16384_array tmm16384_quad_cas tmm16384_quad_lock tmm16384_r32_array tmm16384_r32_quad_cas \
  tmm16384_r32_quad_lock tmm4096_i32_paper spmv4m tmm65536_bf16
python tools/results_table.py gpurun_out/results > gpurun_out/results/results_table.md
bash tools/design_space.sh tmm4096_i32_paper > gpurun_out/design_space.md
bash tools/design_space.sh spmv4m > gpurun_out/design_space_spmv.md

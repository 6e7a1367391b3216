#!/bin/bash
# C3 store ablation + C2 fp32 + C5 (single GPU) bench lines -> gpurun_out/bench_*.json
mkdir -p gpurun_out
for w in tmm16384_array tmm16384_quad_cas tmm16384_quad_lock tmm16384_r32_array tmm16384_r32_quad_cas tmm16384_r32_quad_lock tmm8192_bf16_f32out tmm8192_f32_simt; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 --overhead-reps 10 --no-cpu-baseline > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
  tail -1 gpurun_out/bench_$w.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w', {k:d.get(k) for k in ['value','lp_overhead_pct','t_protected_ms','t_unprotected_ms','t_validate_ms','t_recovery_phase_ms','hash_collisions','hash_error']}, d['roofline']['achieved'], d['roofline']['frac'])" || tail -3 gpurun_out/bench_$w.err
done

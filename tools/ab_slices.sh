# A/B: recovery of 32x32 regions as 128x64 slice tasks (default) vs 128x128 tiles (--recover-tile128)
for w in tmm8192_bf16_r32 tmm16384_r32_array; do
  for i in 1 2; do
    python bench.py --workload $w --no-cpu-baseline --steps 10 > gpurun_out/slices_${w}_on_$i.json 2>/dev/null
    python bench.py --workload $w --no-cpu-baseline --steps 10 --recover-tile128 > gpurun_out/slices_${w}_off_$i.json 2>/dev/null
  done
done

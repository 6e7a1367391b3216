for w in tmm8192_bf16 tmm8192_bf16_r32 tmm16384_array; do
  for i in 1 2; do
    python bench.py --workload $w --no-cpu-baseline --steps 10 > gpurun_out/pair_${w}_on_$i.json 2>/dev/null
    python bench.py --workload $w --no-cpu-baseline --steps 10 --no-pairing > gpurun_out/pair_${w}_off_$i.json 2>/dev/null
  done
done

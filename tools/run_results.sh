#!/bin/bash
# Every bench workload once (single GPU) -> gpurun_out/results/<workload>.json; summary via tools/results_table.py
mkdir -p gpurun_out/results
for w in "$@"; do
  timeout 1200 python bench.py --workload $w --steps 5 --warmup 3 --overhead-reps 10 --no-cpu-baseline > gpurun_out/results/$w.json 2> gpurun_out/results/$w.err
  tail -1 gpurun_out/results/$w.json | cut -c1-200
done

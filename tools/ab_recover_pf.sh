#!/bin/bash
# A/B of the recovery re-execution for 128x128 regions at 8192^3 bf16, 5% failed:
#   paired 128x128 tiles (default) vs 128x64 slice tasks (--recover-slices128);
#   task order: size-sorted snake (default) vs row order (LP_TASK_ORDER=row);
#   L2 prefetch distance LP_TC_PREFETCH (k-blocks, default 0).
mkdir -p gpurun_out
run() {  # label, env, extra args
  env $2 python bench.py --workload tmm8192_bf16 --steps 20 --overhead-reps 2 --no-cpu-baseline $3 \
    | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', d['value'], d['t_recovery_phase_ms'])"
}
for rep in 1 2; do
  run "tile128 lpt     " "LP_TASK_ORDER=lpt" ""
  run "tile128 row     " "LP_TASK_ORDER=row" ""
  run "slices128 lpt   " "LP_TASK_ORDER=lpt" "--recover-slices128"
  run "tile128 lpt pf8 " "LP_TC_PREFETCH=8" ""
done

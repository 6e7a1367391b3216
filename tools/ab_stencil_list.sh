#!/bin/bash
# A/B: list-mode (recovery) stencil: persistent 2 CTAs/SM with the barrier combine (default) vs one region per
# CTA over R CTAs with the split-barrier combine (LP_STENCIL_LIST_ONE=1)
for i in 1 2; do for one in 0 1; do
  LP_STENCIL_LIST_ONE=$one python bench.py --steps 10 --overhead-reps 2 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('one=$one', d['value'], d['t_recovery_phase_ms'], d['t_validate_ms'])"
done; done
LP_STENCIL_LIST_ONE=1 python -m pytest tests/test_gpu_stencil.py -x -q 2>&1 | tail -1

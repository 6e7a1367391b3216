#!/bin/bash
# A/B: list-mode (recovery) stencil grid = n x #SM persistent CTAs
for i in 1 2; do for n in 2 8 32 64; do
  LP_STENCIL_LIST_CTAS=$n python bench.py --steps 10 --overhead-reps 2 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('ctas/SM $n', d['value'], d['t_recovery_phase_ms'], d['t_validate_ms'])"
done; done

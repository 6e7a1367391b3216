#!/bin/bash
# A/B of two liblp builds on the same box: the in-tree one (new) vs build/ab_old/liblp.so (old),
# alternating, same bench arguments.  Usage: bash tools/ab_bench.sh <tag> <bench args...>
tag=$1; shift
for i in 1 2; do
  timeout 600 python bench.py "$@" --no-cpu-baseline > gpurun_out/ab_${tag}_new_$i.json 2> gpurun_out/ab_${tag}_new_$i.err
  timeout 600 python -c "
import runpy, sys
import paper_conf_iiswc_yudhakzs20_b200.lp as l
l.LIB_PATH = 'build/ab_old/liblp.so'
sys.argv = ['bench.py'] + sys.argv[1:]
runpy.run_path('bench.py', run_name='__main__')" "$@" --no-cpu-baseline > gpurun_out/ab_${tag}_old_$i.json 2> gpurun_out/ab_${tag}_old_$i.err
done
for f in gpurun_out/ab_${tag}_*.json; do
  python -c "
import json,sys
d=json.loads(open('$f').read().strip().splitlines()[-1])
print('$f', d['t_protected_ms'], d['t_unprotected_ms'], d['lp_overhead_pct'], d['roofline']['achieved'], d['roofline']['frac'], d['t_validate_ms'], d['value'])" 2>/dev/null || tail -2 gpurun_out/ab_${tag}_*.err
done

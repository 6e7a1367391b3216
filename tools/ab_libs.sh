#!/bin/bash
# A/B of several liblp builds on one box: bash tools/ab_libs.sh <tag> "<lib1> <lib2> ..." <bench args...>
# (each lib path is loaded in place of the in-tree liblp.so; two alternating rounds)
tag=$1; libs=$2; shift 2
for i in 1 2; do
  for L in $libs; do
    n=$(basename $(dirname $L))
    timeout 600 python -c "
import runpy, sys
import paper_conf_iiswc_yudhakzs20_b200.lp as l
l.LIB_PATH = '$L'
sys.argv = ['bench.py'] + sys.argv[1:]
runpy.run_path('bench.py', run_name='__main__')" "$@" --no-cpu-baseline > gpurun_out/ab_${tag}_${n}_$i.json 2> gpurun_out/ab_${tag}_${n}_$i.err
    python -c "
import json
d=json.loads(open('gpurun_out/ab_${tag}_${n}_$i.json').read().strip().splitlines()[-1])
print('$n', $i, d['t_protected_ms'], d['t_unprotected_ms'], d['lp_overhead_pct'], d['roofline']['achieved'], d['roofline']['frac'])" 2>/dev/null || tail -2 gpurun_out/ab_${tag}_${n}_$i.err
  done
done

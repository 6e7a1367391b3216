#!/bin/bash
# A/B: C tile stores evict-first (__stcs, build/abx/cs1) vs plain (build/abx/cs0): body time and DRAM traffic.
mkdir -p gpurun_out
for L in build/abx/cs1/liblp.so build/abx/cs0/liblp.so; do
  n=$(basename $(dirname $L))
  for w in tmm8192_bf16 tmm16384_array; do
    for i in 1 2; do
      timeout 600 python -c "
import runpy, sys
import paper_conf_iiswc_yudhakzs20_b200.lp as l
l.LIB_PATH = '$L'
sys.argv = ['bench.py'] + sys.argv[1:]
runpy.run_path('bench.py', run_name='__main__')" --workload $w --steps 5 --overhead-reps 10 --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); print('$n $w', d['t_protected_ms'], d['t_unprotected_ms'], d['roofline']['frac'], d['clocks']['sm_mhz'])"
    done
  done
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:tmm_tc2 -c 4 python -c "
import runpy, sys
import paper_conf_iiswc_yudhakzs20_b200.lp as l
l.LIB_PATH = '$L'
sys.argv = ['tools/cksum_sweep_kernels.py', '--workload', 'tmm']
runpy.run_path('tools/cksum_sweep_kernels.py', run_name='__main__')" 2>&1 | grep -E "dram__bytes|gpu__time" | head -8 | sed "s/^/$n /"
done

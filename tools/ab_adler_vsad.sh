#!/bin/bash
# A/B: stencil Adler byte sums through dp4a (build/abx/cs1 = in-tree) vs VABSDIFF4 (build/abx/vsad), ncu times
M=gpu__time_duration.sum,sm__inst_executed.sum
for L in build/abx/cs1/liblp.so build/abx/vsad/liblp.so; do
  n=$(basename $(dirname $L))
  for i in 1 2; do
  ncu --metrics $M --clock-control none -k regex:stencil5_ldg --csv python -c "
import runpy, sys
import paper_conf_iiswc_yudhakzs20_b200.lp as l
l.LIB_PATH = '$L'
sys.argv = ['tools/cksum_sweep_kernels.py', '--workload', 'stencil']
runpy.run_path('tools/cksum_sweep_kernels.py', run_name='__main__')" 2>/dev/null | python -c "
import csv, sys
rows=[r for r in csv.reader(sys.stdin) if r and not r[0].startswith('==') and len(r)>10]
h=rows[0]; iid=h.index('ID'); im=h.index('Metric Name'); iv=h.index('Metric Value')
per={}
for r in rows[1:]: per.setdefault(int(r[iid]),{})[r[im]]=float(r[iv].replace(',',''))
L=[per[k] for k in sorted(per)]
t0=L[1]['gpu__time_duration.sum']
print('$n', ' '.join(f'{n}:{100*(L[2*i+1][\"gpu__time_duration.sum\"]/t0-1):+.2f}%' for i,n in enumerate(['twin','MOD','XOR','MX','AD','ALL'])))"
  done
done

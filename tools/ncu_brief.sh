#!/bin/bash
# Key counters of an .ncu-rep (first kernel): time, DRAM, issue, occupancy, top stall reasons.
ncu -i "$1" --page details --csv 2>/dev/null | python -c "
import csv,sys
r=list(csv.reader(sys.stdin)); h=r[0]
si,mi,ui,vi=h.index('Section Name'),h.index('Metric Name'),h.index('Metric Unit'),h.index('Metric Value')
keep={'Duration','Memory Throughput','DRAM Throughput','Executed Ipc Active','Issue Slots Busy','Achieved Occupancy','Registers Per Thread','L2 Hit Rate','L1/TEX Hit Rate','Warp Cycles Per Issued Instruction','Eligible Warps Per Scheduler','Executed Instructions','Mem Busy'}
seen=set()
for x in r[1:]:
  if x[mi] in keep and x[mi] not in seen: seen.add(x[mi]); print(f'{x[mi]:40s} {x[vi]} {x[ui]}')
"
ncu -i "$1" --page raw --csv 2>/dev/null | python -c "
import csv,sys
r=list(csv.reader(sys.stdin)); h,v=r[0],r[2]
out=[]
for i,n in enumerate(h):
  if n.startswith('smsp__average_warp_latency_issue_stalled_') and n.endswith('.ratio'):
    try: out.append((float(v[i]),n.replace('smsp__average_warp_latency_issue_stalled_','').replace('.ratio','')))
    except: pass
  if n.startswith('smsp__average_warps_issue_stalled_') and n.endswith('_per_issue_active.ratio'):
    try: out.append((float(v[i]),n.replace('smsp__average_warps_issue_stalled_','').replace('_per_issue_active.ratio','')))
    except: pass
print('stalls (warps per issue):', ', '.join(f'{b}={a:.2f}' for a,b in sorted(out,reverse=True)[:8]))
"

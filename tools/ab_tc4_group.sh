M=gpu__time_duration.sum,dram__bytes_read.sum,sm__cycles_elapsed.avg.per_second
for g in 1 2 3; do
  LP_TC4_GROUP=$g ncu --metrics $M --clock-control none -k regex:tmm_tc python tools/probe/c5_traffic.py 32768 2>&1 | grep -E "dram__|gpu__time|per_second" | sed "s/^/tc4 G=$g /"
done
for t in 256 128; do for i in 1 2; do LP_TC_TILE=$t python bench.py --workload tmm16384_array --steps 3 --overhead-reps 6 --no-cpu-baseline | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(\"tile$t 16384\", d[\"t_protected_ms\"], d[\"t_unprotected_ms\"], d[\"roofline\"][\"frac\"], d[\"clocks\"][\"sm_mhz\"])"; done; done

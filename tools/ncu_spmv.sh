# ncu --set full of the protected SpMV full run (launch index 2 = the second warm-up step's body)
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 2 -c 1 -o gpurun_out/prof_spmv python bench.py --workload spmv4m --steps 2 --warmup 1 --overhead-reps 2 --no-cpu-baseline > /dev/null 2>&1

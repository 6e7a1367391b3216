# ncu --set full of the protected SpMV full run: in-tree lib (new) and build/ab_old/liblp.so (old)
A="--workload spmv4m --steps 2 --warmup 1 --overhead-reps 2 --no-cpu-baseline"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:spmv_kernel -s 2 -c 1 -o gpurun_out/prof_spmv_new python bench.py $A > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none -k regex:spmv_kernel -s 2 -c 1 -o gpurun_out/prof_spmv_old python -c "
import runpy, sys
import paper_conf_iiswc_yudhakzs20_b200.lp as l
l.LIB_PATH = 'build/ab_old/liblp.so'
sys.argv = ['bench.py'] + sys.argv[1:]
runpy.run_path('bench.py', run_name='__main__')" $A > /dev/null 2>&1

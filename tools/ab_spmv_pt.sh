# A/B: SpMV chunk size (LP_SPMV_PT nnz per thread -> 256 * PT nnz per chunk) x CTAs/SM (LP_SPMV_MINB), scalar
# element mapping; rebuilt on the box, alternating
for cfg in "8 5" "16 4" "16 3" "8 5" "16 4" "12 4"; do
  set -- $cfg
  sed -i "s/^#define LP_SPMV_PT .*/#define LP_SPMV_PT $1/; s/^#define LP_SPMV_MINB .*/#define LP_SPMV_MINB $2/" paper_conf_iiswc_yudhakzs20_b200/csrc/spmv.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  timeout 600 python bench.py --workload spmv4m --no-cpu-baseline --steps 5 > gpurun_out/spmv_PT$1_MB$2.json 2> gpurun_out/spmv_PT$1_MB$2.err
  python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[1], d['t_protected_ms'], d['t_unprotected_ms'], d['lp_overhead_pct'], d['roofline']['frac'], d['value'])" gpurun_out/spmv_PT$1_MB$2.json || tail -3 gpurun_out/spmv_PT$1_MB$2.err
done
sed -i "s/^#define LP_SPMV_PT .*/#define LP_SPMV_PT 8/; s/^#define LP_SPMV_MINB .*/#define LP_SPMV_MINB 5/" paper_conf_iiswc_yudhakzs20_b200/csrc/spmv.cu
make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1

# A/B of the SpMV product-phase element mapping: LP_SPMV_SCALAR=1 (element s*256 + tid, consecutive lanes on
# consecutive elements) vs 0 (4 consecutive elements per thread); rebuilt on the box, alternating
for cfg in "1 5" "0 5" "1 5" "0 5" "1 4"; do
  set -- $cfg
  sed -i "s/^#define LP_SPMV_SCALAR .*/#define LP_SPMV_SCALAR $1/; s/^#define LP_SPMV_MINB .*/#define LP_SPMV_MINB $2/" paper_conf_iiswc_yudhakzs20_b200/csrc/spmv.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  timeout 600 python bench.py --workload spmv4m --no-cpu-baseline --steps 5 > gpurun_out/spmv_S$1_MB$2.json 2> gpurun_out/spmv_S$1_MB$2.err
  python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[1], d['t_protected_ms'], d['t_unprotected_ms'], d['lp_overhead_pct'], d['roofline']['frac'], d['value'])" gpurun_out/spmv_S$1_MB$2.json
done
sed -i "s/^#define LP_SPMV_SCALAR .*/#define LP_SPMV_SCALAR 1/; s/^#define LP_SPMV_MINB .*/#define LP_SPMV_MINB 5/" paper_conf_iiswc_yudhakzs20_b200/csrc/spmv.cu; make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1

# A/B of the SpMV body: next chunk's loads issued early (EARLY=1, register double buffer) vs after the products
# (EARLY=0), with min CTAs/SM (MINB) in the launch bounds; rebuilt on the box, bench.py spmv4m line each.
for cfg in "0 5" "1 4" "1 5" "1 3" "0 4"; do
  set -- $cfg
  sed -i "s/^#define LP_SPMV_EARLY .*/#define LP_SPMV_EARLY $1/; s/^#define LP_SPMV_MINB .*/#define LP_SPMV_MINB $2/" paper_conf_iiswc_yudhakzs20_b200/csrc/spmv.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  timeout 600 python bench.py --workload spmv4m --no-cpu-baseline --steps 5 > gpurun_out/spmv_E$1_MB$2.json 2> gpurun_out/spmv_E$1_MB$2.err
  python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[1], d['t_protected_ms'], d['t_unprotected_ms'], d['lp_overhead_pct'], d['roofline']['frac'], d['value'])" gpurun_out/spmv_E$1_MB$2.json
done

# A/B of the SpMV body: nnz per thread per chunk (PT) and min CTAs/SM in launch bounds (MINB), rebuilt on the box.
set -x
for cfg in "8 4" "16 4" "8 6" "16 3" "4 6"; do
  set -- $cfg
  sed -i "s/^#define LP_SPMV_PT .*/#define LP_SPMV_PT $1/; s/^#define LP_SPMV_MINB .*/#define LP_SPMV_MINB $2/" paper_conf_iiswc_yudhakzs20_b200/csrc/spmv.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  timeout 600 python bench.py --workload spmv4m --no-cpu-baseline --steps 5 > gpurun_out/spmv_PT$1_MB$2.json 2> gpurun_out/spmv_PT$1_MB$2.err
done

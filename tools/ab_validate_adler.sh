# A/B: validate kernel with Adler in the record compiled for 3 vs 4 CTAs/SM (LP_VAL_ADLER_MINB), rebuilt on the box
for mb in 3 4 2; do
  sed -i "s/^#define LP_VAL_ADLER_MINB .*/#define LP_VAL_ADLER_MINB $mb/" paper_conf_iiswc_yudhakzs20_b200/csrc/lp_kernels.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  for w in stencil32768_adler tmm8192_bf16_adler; do
    python bench.py --workload $w --no-cpu-baseline --steps 5 > gpurun_out/va_${mb}_$w.log 2>&1
    python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print('MINB=$mb', sys.argv[1], d['value'], d['t_validate_ms'], d['t_recovery_phase_ms'], d['roofline_validate']['frac'])" gpurun_out/va_${mb}_$w.log
  done
done
sed -i "s/^#define LP_VAL_ADLER_MINB .*/#define LP_VAL_ADLER_MINB 3/" paper_conf_iiswc_yudhakzs20_b200/csrc/lp_kernels.cu

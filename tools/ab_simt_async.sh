# A/B: SIMT TMM operands global -> shared through registers (LP_SIMT_ASYNC=0) vs cp.async (1), each built
# once into build/ab/, 2 interleaved rounds (tmm4096_i32_paper, tmm8192_f32_simt)
mkdir -p build/ab
for mb in 0 1; do
  sed -i "s/^#define LP_SIMT_ASYNC .*/#define LP_SIMT_ASYNC $mb/" paper_conf_iiswc_yudhakzs20_b200/csrc/tmm_simt.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  cp paper_conf_iiswc_yudhakzs20_b200/liblp.so build/ab/liblp_async_$mb.so
done
for round in 1 2; do
  for mb in 0 1; do
    cp build/ab/liblp_async_$mb.so paper_conf_iiswc_yudhakzs20_b200/liblp.so
    for w in tmm4096_i32_paper tmm8192_f32_simt; do
      python bench.py --workload $w --no-cpu-baseline --steps 3 --overhead-reps 4 > gpurun_out/async_${mb}_${w}_$round.log 2>&1
      python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print('ROUND $round ASYNC=$mb $w', d['t_protected_ms'], d['t_unprotected_ms'], d['lp_overhead_pct'], d['roofline']['frac'])" gpurun_out/async_${mb}_${w}_$round.log
    done
  done
done
sed -i "s/^#define LP_SIMT_ASYNC .*/#define LP_SIMT_ASYNC 1/" paper_conf_iiswc_yudhakzs20_b200/csrc/tmm_simt.cu

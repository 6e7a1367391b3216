# A/B: SIMT 128x128-tile builds compiled for 1 CTA/SM (~240 registers) vs 2 CTAs/SM (128 registers, ~50 B spills),
# each built once into build/ab/, run in 2 interleaved rounds (tmm4096_i32_paper, tmm8192_f32_simt)
mkdir -p build/ab
for mb in 2 3; do
  sed -i "s/^#define LP_SIMT_MINB .*/#define LP_SIMT_MINB $mb/" paper_conf_iiswc_yudhakzs20_b200/csrc/tmm_simt.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  cp paper_conf_iiswc_yudhakzs20_b200/liblp.so build/ab/liblp_simt3_$mb.so
done
for round in 1 2; do
  for mb in 2 3; do
    cp build/ab/liblp_simt3_$mb.so paper_conf_iiswc_yudhakzs20_b200/liblp.so
    for w in tmm4096_i32_paper tmm8192_f32_simt; do
      python bench.py --workload $w --no-cpu-baseline --steps 3 --overhead-reps 4 > gpurun_out/simt_${mb}_${w}_$round.log 2>&1
      python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print('ROUND $round MINB=$mb $w', d['t_protected_ms'], d['t_unprotected_ms'], d['lp_overhead_pct'], d['roofline']['frac'])" gpurun_out/simt_${mb}_${w}_$round.log
    done
  done
done
sed -i "s/^#define LP_SIMT_MINB .*/#define LP_SIMT_MINB 2/" paper_conf_iiswc_yudhakzs20_b200/csrc/tmm_simt.cu

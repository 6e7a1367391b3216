# A/B: 3xTF32 kernel with A_hi read from the raw TMA stage (LP_TF32_RAW_HI=1, 4 raw + 2 converted stages of 48 KB)
# vs converted A_hi (0, 3 raw + 2 converted stages of 64 KB); built once each, 3 interleaved rounds
mkdir -p build/ab
for v in 1 0; do
  sed -i "s/^#define LP_TF32_RAW_HI .*/#define LP_TF32_RAW_HI $v/" paper_conf_iiswc_yudhakzs20_b200/csrc/tmm_tf32.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  cp paper_conf_iiswc_yudhakzs20_b200/liblp.so build/ab/liblp_rawhi_$v.so
done
for round in 1 2 3; do
  for v in 1 0; do
    cp build/ab/liblp_rawhi_$v.so paper_conf_iiswc_yudhakzs20_b200/liblp.so
    python bench.py --workload tmm8192_f32 --no-cpu-baseline --steps 5 --overhead-reps 6 > gpurun_out/rawhi_${v}_$round.log 2>&1
    python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print('ROUND $round RAW_HI=$v', d['t_protected_ms'], d['t_unprotected_ms'], d['lp_overhead_pct'], d['roofline']['achieved'], d['clocks']['sm_mhz'], d['t_recovery_phase_ms'])" gpurun_out/rawhi_${v}_$round.log
  done
done
sed -i "s/^#define LP_TF32_RAW_HI .*/#define LP_TF32_RAW_HI 1/" paper_conf_iiswc_yudhakzs20_b200/csrc/tmm_tf32.cu
cp build/ab/liblp_rawhi_1.so paper_conf_iiswc_yudhakzs20_b200/liblp.so

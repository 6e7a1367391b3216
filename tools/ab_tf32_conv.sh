# A/B: converter warps / B-conversion loop form of the 3xTF32 kernel, each variant built once into
# build/ab/, then run in interleaved rounds (the 1 kW power cap makes back-to-back runs drift)
mkdir -p build/ab
V="4:0 8:0 8:1 12:1"
for v in $V; do
  w=${v%:*}; b=${v#*:}
  sed -i "s/^#define LP_TF32_CONV_WARPS .*/#define LP_TF32_CONV_WARPS $w/; s/^#define LP_TF32_BLOOP .*/#define LP_TF32_BLOOP $b/" paper_conf_iiswc_yudhakzs20_b200/csrc/tmm_tf32.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1 && cp paper_conf_iiswc_yudhakzs20_b200/liblp.so build/ab/liblp_$w_$b.so
  cp paper_conf_iiswc_yudhakzs20_b200/liblp.so build/ab/liblp_${w}_${b}.so
done
for round in 1 2 3; do
  for v in $V; do
    w=${v%:*}; b=${v#*:}
    cp build/ab/liblp_${w}_${b}.so paper_conf_iiswc_yudhakzs20_b200/liblp.so
    python bench.py --workload tmm8192_f32 --no-cpu-baseline --steps 5 --overhead-reps 6 > gpurun_out/tf32_${w}_${b}_$round.log 2>&1
    python -c "import json,sys; d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print('ROUND $round CONV_WARPS=$w BLOOP=$b', d['t_protected_ms'], d['t_unprotected_ms'], d['lp_overhead_pct'], d['roofline']['achieved'], d['clocks']['sm_mhz'])" gpurun_out/tf32_${w}_${b}_$round.log
  done
done
sed -i "s/^#define LP_TF32_CONV_WARPS .*/#define LP_TF32_CONV_WARPS 8/; s/^#define LP_TF32_BLOOP .*/#define LP_TF32_BLOOP 0/" paper_conf_iiswc_yudhakzs20_b200/csrc/tmm_tf32.cu
make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1

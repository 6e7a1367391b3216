# A/B: output store flavour of the TMA-fed stencil form (the list-mode recovery): .cs (0) vs .cg (1)
mkdir -p build/ab
for v in 0 1; do
  sed -i "s/^#define LP_STENCIL_TMA_ST_CG .*/#define LP_STENCIL_TMA_ST_CG $v/" paper_conf_iiswc_yudhakzs20_b200/csrc/stencil.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  cp paper_conf_iiswc_yudhakzs20_b200/liblp.so build/ab/liblp_tst_$v.so
done
for round in 1 2 3; do
  for v in 0 1; do
    cp build/ab/liblp_tst_$v.so paper_conf_iiswc_yudhakzs20_b200/liblp.so
    for f in 0.1 0.5; do python tools/run_stencil_recover_once.py $f | sed "s/^/ROUND $round CG=$v frac=$f /"; done
  done
done
sed -i "s/^#define LP_STENCIL_TMA_ST_CG .*/#define LP_STENCIL_TMA_ST_CG 0/" paper_conf_iiswc_yudhakzs20_b200/csrc/stencil.cu
cp build/ab/liblp_tst_0.so paper_conf_iiswc_yudhakzs20_b200/liblp.so

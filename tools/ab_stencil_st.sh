# A/B: store flavour of the stencil LDG form (LP_STENCIL_ST: 0 st.global.cs, 1 plain, 2 .cg, 3 L1::no_allocate),
# built once each, 2 interleaved rounds of tools/ab_stencil_tma.py (masks 3 and 4) + the default bench value
mkdir -p build/ab
for v in 0 1 2 3; do
  sed -i "s/^#define LP_STENCIL_ST .*/#define LP_STENCIL_ST $v/" paper_conf_iiswc_yudhakzs20_b200/csrc/stencil.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  cp paper_conf_iiswc_yudhakzs20_b200/liblp.so build/ab/liblp_st_$v.so
done
for round in 1 2; do
  for v in 0 1 2 3; do
    cp build/ab/liblp_st_$v.so paper_conf_iiswc_yudhakzs20_b200/liblp.so
    LP_TAG=ST$v python tools/ab_stencil_tma.py 3 4 | sed "s/^/ROUND $round ST=$v /"
  done
done
sed -i "s/^#define LP_STENCIL_ST .*/#define LP_STENCIL_ST 0/" paper_conf_iiswc_yudhakzs20_b200/csrc/stencil.cu
cp build/ab/liblp_st_0.so paper_conf_iiswc_yudhakzs20_b200/liblp.so

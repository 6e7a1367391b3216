# A/B: the stencil's 4-B edge-column loads (LP_STENCIL_EDGE_LD: 0 ld.global.nc, 1 .nc.L2::64B, 2 ld.global,
# 3 .nc.L1::no_allocate), rebuilt on the box: list-mode recovery time + DRAM bytes, full-run time.
for e in 0 1 2 3; do
  sed -i "s/^#define LP_STENCIL_EDGE_LD .*/#define LP_STENCIL_EDGE_LD $e/" paper_conf_iiswc_yudhakzs20_b200/csrc/stencil.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  echo "EDGE_LD=$e"; python tools/run_stencil_recover_once.py
  timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum --clock-control none -k regex:stencil5_ldg -s 1 -c 1 python tools/run_stencil_recover_once.py 2>&1 | grep -E "dram__|gpu__time|lts__"
  python tools/ab_stencil_tma.py 3
done
sed -i "s/^#define LP_STENCIL_EDGE_LD .*/#define LP_STENCIL_EDGE_LD 0/" paper_conf_iiswc_yudhakzs20_b200/csrc/stencil.cu

# build the normal and the probe library, run both, compare output bits
mkdir -p build/ab
for p in 0 1; do
  sed -i "s/^#define LP_TF32_RAW_HI_PROBE .*/#define LP_TF32_RAW_HI_PROBE $p/" paper_conf_iiswc_yudhakzs20_b200/csrc/tmm_tf32.cu
  make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1
  python tools/probe/tf32_raw_hi.py gpurun_out/tf32_probe_$p.npy
done
sed -i "s/^#define LP_TF32_RAW_HI_PROBE .*/#define LP_TF32_RAW_HI_PROBE 0/" paper_conf_iiswc_yudhakzs20_b200/csrc/tmm_tf32.cu
python -c "
import numpy as np
a=np.load('gpurun_out/tf32_probe_0.npy'); b=np.load('gpurun_out/tf32_probe_1.npy')
print('identical bits:', np.array_equal(a.view(np.uint32), b.view(np.uint32)), 'max abs diff', float(np.abs(a-b).max()))"

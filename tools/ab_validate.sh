# A/B of the validate kernel: the working tree vs another lp_kernels.cu (AB_OLD_SRC, e.g. from
# `git show <rev>:paper_conf_iiswc_yudhakzs20_b200/csrc/lp_kernels.cu > tools/_ab_old.cu`), built on the box.
set -x
OLD=${AB_OLD_SRC:-tools/_ab_old.cu}
rm -rf /tmp/abold && mkdir -p /tmp/abold && cp -r paper_conf_iiswc_yudhakzs20_b200 include Makefile /tmp/abold/
cp "$OLD" /tmp/abold/paper_conf_iiswc_yudhakzs20_b200/csrc/lp_kernels.cu
(cd /tmp/abold && make -j16 paper_conf_iiswc_yudhakzs20_b200/liblp.so > /dev/null 2>&1)
for i in 1 2; do
python tools/validate_sweep.py > gpurun_out/vs_new_$i.txt 2>&1
LP_AB_LIB=/tmp/abold/paper_conf_iiswc_yudhakzs20_b200/liblp.so python tools/validate_sweep.py > gpurun_out/vs_old_$i.txt 2>&1
done

timeout 600 python -m pytest tests/test_gpu_tmm.py tests/test_gpu_edges.py -x -q > gpurun_out/slice_tests.log 2>&1; echo EXIT $? >> gpurun_out/slice_tests.log
for f in 0.003 0.005; do
  bash tools/ab_libs.sh g$f "build/ab/g4/liblp.so build/ab/gdyn/liblp.so" --workload tmm8192_bf16_r32 --inject-frac $f --steps 10
done

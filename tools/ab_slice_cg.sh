# A/B: slice ids row-major (gdyn build) vs column-group-major in groups of 32 slice columns (cg32 build)
timeout 600 python -m pytest tests/test_gpu_tmm.py tests/test_gpu_edges.py -x -q > gpurun_out/slice_tests.log 2>&1; echo EXIT $? >> gpurun_out/slice_tests.log
timeout 600 python -m pytest tests/test_gpu_fullsize.py -x -q -k "r32 or slice" > gpurun_out/slice_full.log 2>&1; echo EXIT $? >> gpurun_out/slice_full.log
for w in tmm8192_bf16_r32 tmm16384_r32_array; do
  bash tools/ab_libs.sh cg_$w "build/ab/gdyn/liblp.so build/ab/cg32/liblp.so" --workload $w --steps 10
done

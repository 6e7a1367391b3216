# A/B: list-mode re-execution launched with programmatic dependent launch (pdl build) vs plain launch (base)
timeout 600 python -m pytest tests/test_gpu_tmm.py tests/test_gpu_edges.py tests/test_gpu_graph.py -x -q > gpurun_out/pdl_tests.log 2>&1; echo EXIT $? >> gpurun_out/pdl_tests.log
for w in tmm8192_bf16 tmm8192_bf16_r32; do
  bash tools/ab_libs.sh pdl_$w "build/ab/base/liblp.so build/ab/pdl/liblp.so" --workload $w --steps 10
done

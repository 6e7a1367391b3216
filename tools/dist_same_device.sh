#!/bin/bash
# The N>1 bench path on a 1-GPU box: 2 ranks over gloo, both on cuda:0 (timing meaningless; checks the
# sharding, barriers, count all-reduce, max-over-ranks reduction and the JSON line).
P="python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533"
timeout 600 $P bench.py --gpus 2 --steps 2 --warmup 3 --overhead-reps 4 --dist-backend gloo --same-device > gpurun_out/dist2_default.json 2> gpurun_out/dist2_default.err
timeout 900 $P bench.py --gpus 2 --steps 2 --warmup 3 --overhead-reps 2 --no-cpu-baseline --workload tmm65536_bf16 --dist-backend gloo --same-device > gpurun_out/dist2_c5.json 2> gpurun_out/dist2_c5.err
timeout 300 $P bench.py --impl reference --gpus 2 --steps 2 --warmup 1 > gpurun_out/dist2_ref.json 2> gpurun_out/dist2_ref.err
for f in dist2_default dist2_c5 dist2_ref; do echo "== $f"; tail -c 600 gpurun_out/$f.json; tail -3 gpurun_out/$f.err; done

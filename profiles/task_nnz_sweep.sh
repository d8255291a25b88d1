#!/bin/bash
# SR_TASK_NNZ sweep of the phase-S row-group task size on the final kernels (C2, K=128 and K=32).
mkdir -p gpurun_out
for K in 128 32; do for T in ${TS:-64 96 128 192 256}; do
  SR_TASK_NNZ=$T timeout 300 python bench.py --K $K --steps 20 --warmup 5 --e2e-steps 0 --no-cpu-baseline \
    > gpurun_out/tn_K${K}_T${T}.json 2> gpurun_out/tn_K${K}_T${T}.err; echo "K=$K T=$T rc=$?"
done; done

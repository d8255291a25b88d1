#!/bin/bash
# session-3 GPU batch: new tests, dense threshold sweep under the task kernels, CF loop, slow tests
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m "gpu and not slow" -q --timeout 600 > gpurun_out/s3_pytest_gpu.log 2>&1; tail -3 gpurun_out/s3_pytest_gpu.log
for dm in 1000000 64 16 8; do
  timeout 300 python bench.py --no-cpu-baseline --e2e-steps 0 --dense-min $dm > gpurun_out/s3_dm$dm.json 2> gpurun_out/s3_dm$dm.err; echo "dm $dm rc=$?"
done
timeout 300 python bench.py --no-cpu-baseline --e2e-steps 0 --mode off > gpurun_out/s3_off.json 2> gpurun_out/s3_off.err; echo "off rc=$?"
timeout 600 python examples/cf_gd.py > gpurun_out/s3_cf.json 2> gpurun_out/s3_cf.err; echo "cf rc=$?"
timeout 1500 python -m pytest tests -m "slow" -q --timeout 1400 > gpurun_out/s3_pytest_slow.log 2>&1; tail -3 gpurun_out/s3_pytest_slow.log

#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m "gpu and not slow" -q --timeout 600 > gpurun_out/s3b_pytest_gpu.log 2>&1; tail -2 gpurun_out/s3b_pytest_gpu.log
bash profiles/sweep.sh s3b 0 "128" "-" "SR_SPARSE_VARIANT=9" "SR_SPARSE_VARIANT=10"
bash profiles/sweep.sh s3b 0 "32" "-" "SR_SPARSE_VARIANT=8" "SR_SPARSE_VARIANT=9" "SR_SPARSE_VARIANT=10"
timeout 900 python examples/cf_gd.py > gpurun_out/s3b_cf.json 2> gpurun_out/s3b_cf.err; echo "cf rc=$?"

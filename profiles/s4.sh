#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -k "engines" --timeout 800 > gpurun_out/s4_pytest.log 2>&1; tail -2 gpurun_out/s4_pytest.log
BENCH_ARGS="--ops spmm" bash profiles/sweep.sh s4 0 "32" "-" "SR_SPARSE_VARIANT=8" "SR_SPARSE_VARIANT=9"
bash profiles/other_configs.sh r01d

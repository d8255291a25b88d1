#!/bin/bash
# quick GPU iteration: gpu tests (not slow) + one bench run -> gpurun_out/$1.json
tag=${1:-q}; shift
timeout 600 python -m pytest tests -m "gpu and not slow" -q --timeout 300 2>&1 | grep -E "Error|passed|failed" | head -5
python bench.py --no-cpu-baseline --e2e-steps 0 "$@" > gpurun_out/$tag.json 2> gpurun_out/$tag.err; tail -3 gpurun_out/$tag.err

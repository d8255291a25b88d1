#!/bin/bash
# GPU iteration helper (under gpurun): optional gpu tests, then one bench line per
# environment variant and K.  Usage: bash profiles/sweep.sh <tag> <run_tests 0|1> "<K list>" "<variant>"...
# A variant is a space-separated list of VAR=value settings ("-" = defaults), e.g. "SR_STREAM=4".
tag=$1; tests=$2; klist=$3; shift 3
mkdir -p gpurun_out
if [ "$tests" = "1" ]; then
  timeout 900 python -m pytest tests -m "gpu and not slow" -q -x --timeout 300 2>&1 | tail -15
fi
for v in "$@"; do
  vt=$(echo "$v" | tr ' =' '__')
  for K in $klist; do
    if [ "$v" = "-" ]; then e=""; else e="$v"; fi
    env $e timeout 300 python bench.py --no-cpu-baseline --e2e-steps 0 --K $K $BENCH_ARGS \
      > gpurun_out/${tag}_${vt}_K$K.json 2> gpurun_out/${tag}_${vt}_K$K.err
    echo "$v K=$K rc=$? $(tail -c 300 gpurun_out/${tag}_${vt}_K$K.err | tail -1)"
  done
done

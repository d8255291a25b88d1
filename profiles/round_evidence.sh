#!/bin/bash
# Round-end evidence (under gpurun): gpu tests, smoke, the default bench line (K=128), the
# K=32 line, the reference arm, the ncu launch list of the default bench and one
# `ncu --set full` capture of each phase kernel.  Usage: bash profiles/round_evidence.sh <tag>
tag=${1:-r01}
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 > gpurun_out/${tag}_pytest_gpu.log 2>&1; tail -3 gpurun_out/${tag}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${tag}_smoke.log 2>&1; tail -1 gpurun_out/${tag}_smoke.log
timeout 600 python bench.py > gpurun_out/${tag}_bench.json 2> gpurun_out/${tag}_bench.err; echo "bench rc=$?"
timeout 600 python bench.py --K 32 > gpurun_out/${tag}_bench_k32.json 2> gpurun_out/${tag}_bench_k32.err; echo "bench k32 rc=$?"
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/${tag}_bench_ref.json 2> gpurun_out/${tag}_bench_ref.err; echo "ref rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${tag}_launches.csv \
  python bench.py --steps 2 --warmup 1 --min-warm-s 0 --e2e-steps 0 --no-cpu-baseline > /dev/null 2>&1; echo "launches rc=$?"
timeout 900 bash profiles/ncu_capture.sh ${tag}k128 "spmm_task|sddmm_task|spmm_dense|sddmm_dense" 4 > /dev/null 2>&1; echo "ncu k128 rc=$?"
timeout 900 bash profiles/ncu_capture.sh ${tag}k32 "spmm_task|sddmm_task|spmm_dense|sddmm_dense" 4 --K 32 > /dev/null 2>&1; echo "ncu k32 rc=$?"

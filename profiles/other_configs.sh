#!/bin/bash
# bench lines of the non-headline configs (parity-test cases), one op mix each
mkdir -p gpurun_out
tag=${1:-r01d}
timeout 600 python bench.py --config banded --no-cpu-baseline --e2e-steps 0 > gpurun_out/${tag}_banded.json 2> gpurun_out/${tag}_banded.err; echo "banded rc=$?"
timeout 600 python bench.py --config gnn --ops spmm --no-cpu-baseline --e2e-steps 0 > gpurun_out/${tag}_gnn.json 2> gpurun_out/${tag}_gnn.err; echo "gnn rc=$?"
timeout 600 python bench.py --config gnn --ops spmm --mode off --no-cpu-baseline --e2e-steps 0 > gpurun_out/${tag}_gnn_off.json 2> gpurun_out/${tag}_gnn_off.err; echo "gnn off rc=$?"
timeout 900 python bench.py --config cf --ops sddmm --no-cpu-baseline --e2e-steps 0 > gpurun_out/${tag}_cf.json 2> gpurun_out/${tag}_cf.err; echo "cf rc=$?"
timeout 600 python bench.py --config cf --ops sddmm --mode off --no-cpu-baseline --e2e-steps 0 > gpurun_out/${tag}_cf_off.json 2> gpurun_out/${tag}_cf_off.err; echo "cf off rc=$?"

# round 2, session c: GPU tests (incl. sanitizers, C2 whole output), bench line, other configs
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
timeout 2400 python -m pytest tests -m "gpu and not slow" -q -x 2>&1 | tail -25 > $O/r02c_pytest_fast.log
SR_DEBUG_CLUSTER=1 timeout 1200 python bench.py > $O/r02c_bench.json 2> $O/r02c_bench.err
timeout 1800 python -m pytest tests/test_gpu_parity.py -m slow -q -x -k "rmat_whole_output or (plan_bench_params and (rmat or banded))" 2>&1 | tail -15 > $O/r02c_pytest_slow.log
SR_DEBUG_CLUSTER=1 timeout 900 python bench.py --config gnn --ops spmm --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --simulate-world 8 > $O/r02c_bench_gnn.json 2> $O/r02c_bench_gnn.err
SR_DEBUG_CLUSTER=1 timeout 900 python bench.py --config cf --ops sddmm --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --simulate-world 8 > $O/r02c_bench_cf.json 2> $O/r02c_bench_cf.err
timeout 900 python bench.py --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --simulate-world 8 --extra-K "" > $O/r02c_bench_sim8.json 2> $O/r02c_bench_sim8.err
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/r02c_smoke.log 2>&1
tail -3 $O/r02c_pytest_fast.log $O/r02c_pytest_slow.log $O/r02c_smoke.log

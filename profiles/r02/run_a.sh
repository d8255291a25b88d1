set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1500 python -m pytest tests -m "gpu and not slow" -x -q 2>&1 | tail -15 > gpurun_out/r02a_pytest.log
SR_DEBUG_CLUSTER=1 timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/r02a_bench_rmat.json 2> gpurun_out/r02a_bench_rmat.err
SR_DEBUG_CLUSTER=1 timeout 900 python bench.py --config banded --steps 10 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/r02a_bench_banded.json 2> gpurun_out/r02a_bench_banded.err
tail -3 gpurun_out/r02a_pytest.log

# round 2, session x: the full GPU test suite on the current code (incl. full-size configs)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
O=gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/r02x_smoke.log 2>&1; echo smoke $?
start=$(date +%s)
timeout 3000 python -m pytest tests -m gpu -q --durations=15 2>&1 | tail -30 > $O/r02x_pytest_gpu.log
echo "gpu tests wall $(( $(date +%s) - start )) s" >> $O/r02x_pytest_gpu.log
tail -4 $O/r02x_pytest_gpu.log

# round 2, session r: ticket-driven SDDMM task kernel at K=128 only (launch order elsewhere) —
# parity incl. repeated launches, sanitizers, bench x2
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_sanitizers.py -m "gpu and not slow" -q -x 2>&1 | tail -3 > $O/r02r_pt.log
B="python bench.py --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --plan-cache /tmp/c2.plan"
timeout 900 $B > $O/r02r_bench1.json 2> $O/r02r_bench1.err
timeout 900 $B > $O/r02r_bench2.json 2> $O/r02r_bench2.err
cat $O/r02r_pt.log

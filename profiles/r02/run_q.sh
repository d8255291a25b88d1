# round 2, session q: ticket-driven task kernels (warps draw tasks until they run out) — parity,
# bench, ncu of the phase-S kernels
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m "gpu and not slow" -q -x 2>&1 | tail -3 > $O/r02q_pt.log
B="python bench.py --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --plan-cache /tmp/c2.plan"
timeout 900 $B > $O/r02q_bench1.json 2> $O/r02q_bench1.err
timeout 900 $B > $O/r02q_bench2.json 2> $O/r02q_bench2.err
NB="python bench.py --steps 2 --warmup 3 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none --plan-cache /tmp/c2.plan"
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:task_kernel -s 6 -c 2 -o $O/r02q_prof_k128 $NB > $O/r02q_ncu_k128.log 2>&1
cat $O/r02q_pt.log

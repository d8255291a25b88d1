# round 2, session l: two-entries-per-step SpMM task kernel (SR_SPMM_PAIR), tagged-cursor pipelined Alg 3
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
for v in 1 2 3; do SR_SPMM_PAIR=$v timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "k_sweep or long_rows or tiny or strided or empty or unsorted or set_values" 2>&1 | tail -2 > $O/r02l_pt_pair$v.log; done
B="python bench.py --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --ops spmm --plan-cache /tmp/c2.plan"
for v in 0 1 2 3 0; do SR_SPMM_PAIR=$v timeout 900 $B > $O/r02l_pair$v.json 2> $O/r02l_pair$v.err; done
SR_DEBUG_REORDER=1 SR_DEBUG_CLUSTER=1 timeout 900 python bench.py --steps 5 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none > $O/r02l_pre.json 2> $O/r02l_pre.err
SR_DEBUG_REORDER=1 timeout 900 python bench.py --steps 5 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none > $O/r02l_pre2.json 2> $O/r02l_pre2.err
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "plan or worked or shard" 2>&1 | tail -3 > $O/r02l_pytest.log
grep -h sr_reorder $O/r02l_*.err; tail -1 $O/r02l_pt_pair*.log

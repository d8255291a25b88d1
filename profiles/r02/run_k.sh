# round 2, session k: SDDMM X fragment from shared memory (SR_SDDMM_XS), pipelined Alg 3 (8 threads) check
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
B="python bench.py --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --ops sddmm --plan-cache /tmp/c2.plan"
SR_DEBUG_REORDER=1 timeout 900 $B > $O/r02k_xs0.json 2> $O/r02k_xs0.err
for v in 1 2 0; do SR_SDDMM_XS=$v timeout 900 $B > $O/r02k_xs${v}b.json 2> $O/r02k_xs${v}b.err; done
SR_DEBUG_REORDER=1 SR_DEBUG_CLUSTER=1 timeout 900 python bench.py --steps 5 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none > $O/r02k_pre.json 2> $O/r02k_pre.err
for v in 1 2; do SR_SDDMM_XS=$v timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "k_sweep or long_rows or tiny" 2>&1 | tail -2 > $O/r02k_pt_xs$v.log; done
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "plan or worked or shard or trial" 2>&1 | tail -3 > $O/r02k_pytest.log
grep sr_reorder $O/r02k_*.err

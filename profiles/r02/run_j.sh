# round 2, session j: preprocessing breakdown (pipelined Alg 3, pool trim on/off)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
B="python bench.py --steps 5 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none"
SR_DEBUG_REORDER=1 SR_DEBUG_CLUSTER=1 SR_DEBUG_LSH=1 timeout 900 $B > $O/r02j_dbg.json 2> $O/r02j_dbg.err
SR_DEBUG_REORDER=1 timeout 900 $B > $O/r02j_trim.json 2> $O/r02j_trim.err
SR_DEBUG_REORDER=1 SR_POOL_KEEP=1 timeout 900 $B > $O/r02j_keep.json 2> $O/r02j_keep.err
SR_DEBUG_REORDER=1 SR_CLUSTER_NOPIPE=1 timeout 900 $B > $O/r02j_nopipe.json 2> $O/r02j_nopipe.err
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "plan or cluster or worked or shard or trial" 2>&1 | tail -3 > $O/r02j_pytest.log
grep sr_reorder $O/r02j_*.err

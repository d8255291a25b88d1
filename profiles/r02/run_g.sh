# round 2, session g: speculative Alg 3 + pooled LSH temporaries (C2 preprocessing), chunked register tiles (C4)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
timeout 2400 python -m pytest tests -m "gpu and not slow" -q -x 2>&1 | tail -25 > $O/r02g_pytest_fast.log
SR_DEBUG_LSH=1 SR_DEBUG_CLUSTER=1 timeout 900 python bench.py --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K "" > $O/r02g_bench_dbg.json 2> $O/r02g_bench_dbg.err
timeout 900 python bench.py --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K "" > $O/r02g_bench.json 2> $O/r02g_bench.err
B="python bench.py --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0"
timeout 900 $B --config gnn --ops spmm --panel-rows 8 --dense-min 2 > $O/r02g_rt_gnn.json 2> $O/r02g_rt_gnn.err
timeout 900 $B --config gnn --ops spmm --panel-rows 8 --dense-min 3 > $O/r02g_rt_gnn3.json 2> $O/r02g_rt_gnn3.err
timeout 900 $B --config gnn --ops spmm > $O/r02g_gnn.json 2> $O/r02g_gnn.err
timeout 900 $B --config rmat --panel-rows 8 --dense-min 2 > $O/r02g_rt_rmat.json 2> $O/r02g_rt_rmat.err
SR_DEBUG_CLUSTER=1 timeout 900 $B --config cf --ops sddmm > $O/r02g_cf.json 2> $O/r02g_cf.err
tail -3 $O/r02g_pytest_fast.log

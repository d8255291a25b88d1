# round 2, session f: register-tile variants (SR_RT_VARIANT) + hub panels on the TMA engine; per-band LSH restored with
# the warp kernel for long Jaccard pairs
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
timeout 2400 python -m pytest tests -m "gpu and not slow" -q -x 2>&1 | tail -25 > $O/r02f_pytest_fast.log
SR_DEBUG_LSH=1 SR_DEBUG_CLUSTER=1 timeout 900 python bench.py --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K "" > $O/r02f_bench.json 2> $O/r02f_bench.err
timeout 900 python bench.py --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K "" > $O/r02f_bench_nodbg.json 2> $O/r02f_bench_nodbg.err
B="python bench.py --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --panel-rows 8 --dense-min 2"
for v in 0 1 2 3; do
  SR_RT_VARIANT=$v timeout 900 $B --config gnn --ops spmm --plan-cache /tmp/gnn_p8.plan > $O/r02f_rt_gnn_v$v.json 2> $O/r02f_rt_gnn_v$v.err
  SR_RT_VARIANT=$v timeout 900 $B --config rmat --ops spmm --plan-cache /tmp/rmat_p8.plan > $O/r02f_rt_rmat_v$v.json 2> $O/r02f_rt_rmat_v$v.err
done
timeout 900 $B --config cf --ops sddmm --plan-cache /tmp/cf_p8.plan > $O/r02f_rt_cf.json 2> $O/r02f_rt_cf.err
timeout 900 $B --config rmat --ops sddmm --plan-cache /tmp/rmat_p8.plan > $O/r02f_rt_rmat_sddmm.json 2> $O/r02f_rt_rmat_sddmm.err
tail -3 $O/r02f_pytest_fast.log

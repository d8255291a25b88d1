# round 2, session h: register-tile jump-table variants on C4; full-size parity of C4 / C5 at bench parameters
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
B="python bench.py --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --config gnn --ops spmm --panel-rows 8"
for dm in 2 3; do for v in 0 4 5; do
  SR_RT_VARIANT=$v timeout 900 $B --dense-min $dm --plan-cache /tmp/gnn_p8_dm$dm.plan > $O/r02h_rt_gnn_dm${dm}_v$v.json 2> $O/r02h_rt_gnn_dm${dm}_v$v.err
done; done
start=$(date +%s)
timeout 3000 python -m pytest tests/test_gpu_parity.py -m slow -q -k "gnn or cf" --durations=10 2>&1 | tail -20 > $O/r02h_pytest_slow.log
echo "slow tests wall $(( $(date +%s) - start )) s" >> $O/r02h_pytest_slow.log
tail -5 $O/r02h_pytest_slow.log

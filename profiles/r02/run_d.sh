# round 2, session d: fast GPU tests + sanitizers, C2 bench (one-pass LSH, lazy identity plan,
# parallel plan build), and the dense-tile statistics of 8- and 16-row panels (register-tile study)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
timeout 2400 python -m pytest tests -m "gpu and not slow" -q 2>&1 | tail -25 > $O/r02d_pytest_fast.log
SR_DEBUG_CLUSTER=1 timeout 1200 python bench.py --no-cpu-baseline --no-oracle-reorder > $O/r02d_bench.json 2> $O/r02d_bench.err
for cfg in rmat gnn cf; do
  ops=spmm,sddmm; [ $cfg = gnn ] && ops=spmm; [ $cfg = cf ] && ops=sddmm
  for pr in 8 16; do
    timeout 900 python bench.py --config $cfg --ops $ops --panel-rows $pr --dense-min 2 --auto-dense-min 100000 --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K "" > $O/r02d_tiles_${cfg}_p$pr.json 2> $O/r02d_tiles_${cfg}_p$pr.err
  done
done
tail -3 $O/r02d_pytest_fast.log

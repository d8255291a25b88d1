# round 2, session e: register-tile phase D (panels of 8 rows) — parity + perf on C2/C4/C5; LSH phase timing
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
timeout 2400 python -m pytest tests -m "gpu and not slow" -q 2>&1 | tail -25 > $O/r02e_pytest_fast.log
SR_DEBUG_LSH=1 SR_DEBUG_CLUSTER=1 timeout 900 python bench.py --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K "" > $O/r02e_bench.json 2> $O/r02e_bench.err
for cfg in rmat gnn cf; do
  ops=spmm,sddmm; [ $cfg = gnn ] && ops=spmm; [ $cfg = cf ] && ops=sddmm
  for dm in 2 3; do
    timeout 900 python bench.py --config $cfg --ops $ops --panel-rows 8 --dense-min $dm --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 > $O/r02e_rt_${cfg}_dm$dm.json 2> $O/r02e_rt_${cfg}_dm$dm.err
  done
done
tail -3 $O/r02e_pytest_fast.log

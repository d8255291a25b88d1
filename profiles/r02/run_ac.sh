# round 2, session ac: final evidence of the round's code (whole-panel phase-D units, SDDMM step skipping) — full GPU test suite, smoke, bench (both arms),
# ncu --set full of the phase-S kernels (K=128, K=32), launch list, Alg 3 block-size sweep, shard simulation
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
python -c "import bench; print(bench.kernel_source_sig())" > $O/r02ac_kernel_sig.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/r02ac_smoke.log 2>&1
timeout 900 python bench.py > $O/r02ac_bench.json 2> $O/r02ac_bench.err
timeout 900 python bench.py --impl reference > $O/r02ac_bench_ref.json 2> $O/r02ac_bench_ref.err
NB="python bench.py --steps 2 --warmup 3 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none --plan-cache /tmp/c2.plan"
timeout 600 $NB > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:task_kernel -s 6 -c 2 -o $O/r02ac_prof_k128 $NB > $O/r02ac_ncu_k128.log 2>&1
for r in k128; do ncu -i $O/r02ac_prof_$r.ncu-rep --page raw --csv > $O/ncu_r02ac_${r}_raw.csv 2>/dev/null; ncu -i $O/r02ac_prof_$r.ncu-rep --page details --csv > $O/ncu_r02ac_${r}_details.csv 2>/dev/null; rm -f $O/r02ac_prof_$r.ncu-rep; done
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:task_kernel -s 6 -c 2 -o $O/r02ac_prof_k32 $NB --K 32 > $O/r02ac_ncu_k32.log 2>&1
for r in k32; do ncu -i $O/r02ac_prof_$r.ncu-rep --page raw --csv > $O/ncu_r02ac_${r}_raw.csv 2>/dev/null; ncu -i $O/r02ac_prof_$r.ncu-rep --page details --csv > $O/ncu_r02ac_${r}_details.csv 2>/dev/null; rm -f $O/r02ac_prof_$r.ncu-rep; done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r02ac_launches.csv python bench.py --steps 2 --warmup 1 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none > /dev/null 2>&1
SR_DEBUG_REORDER=1 SR_DEBUG_CLUSTER=1 SR_DEBUG_LSH=1 timeout 900 python bench.py --steps 5 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none > $O/r02ac_pre.json 2> $O/r02ac_pre.err
for cfg in gnn cf banded; do
  ops=spmm,sddmm; [ $cfg = gnn ] && ops=spmm; [ $cfg = cf ] && ops=sddmm
  SR_DEBUG_REORDER=1 timeout 1200 python bench.py --config $cfg --ops $ops --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 > $O/r02ac_$cfg.json 2> $O/r02ac_$cfg.err
done
for w in 2 4 8; do timeout 900 python bench.py --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none --simulate-world $w --plan-cache /tmp/c2.plan > $O/r02ac_sim$w.json 2> $O/r02ac_sim$w.err; done
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"spmm_dense|spmm_task" -c 2 -o $O/r02ac_prof_gnn python bench.py --config gnn --ops spmm --steps 1 --warmup 1 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --plan-cache /tmp/gnn_ac.plan > $O/r02ac_ncu_gnn.log 2>&1
ncu -i $O/r02ac_prof_gnn.ncu-rep --page raw --csv > $O/ncu_r02ac_gnn_raw.csv 2>/dev/null; rm -f $O/r02ac_prof_gnn.ncu-rep
du -sh $O
# (the full GPU suite ran in the first attempt of this session: profiles/r02/r02ac_pytest_gpu.log)

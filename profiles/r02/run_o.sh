# round 2, session o: evidence of the current code after the container re-creation — smoke, bench
# (both arms), ncu --set full of the phase-S kernels (K=128, K=32) + traffic records, launch list
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
python -c "import bench; print(bench.kernel_source_sig())" > $O/r02o_kernel_sig.txt
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/r02o_smoke.log 2>&1; echo smoke $?
timeout 900 python bench.py > $O/r02o_bench.json 2> $O/r02o_bench.err; echo bench $?
timeout 900 python bench.py --impl reference > $O/r02o_bench_ref.json 2> $O/r02o_bench_ref.err
NB="python bench.py --steps 2 --warmup 3 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none --plan-cache /tmp/c2.plan"
timeout 600 $NB > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:task_kernel -s 6 -c 2 -o $O/r02o_prof_k128 $NB > $O/r02o_ncu_k128.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:task_kernel -s 6 -c 2 -o $O/r02o_prof_k32 $NB --K 32 > $O/r02o_ncu_k32.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r02o_launches.csv python bench.py --steps 2 --warmup 1 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none > /dev/null 2>&1
tail -3 $O/r02o_smoke.log; head -c 400 $O/r02o_bench.json

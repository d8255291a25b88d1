# round 2, session s: memcheck log of the ticket-driven kernel; ncu of the phase-D TMA engine and
# phase S on C4 (GNN) with 64-row panels, dense_min 8
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
timeout 900 compute-sanitizer --tool memcheck --leak-check no --print-limit 10 python tests/sanitizer_cases.py > $O/r02s_memcheck.log 2>&1; echo memcheck $?
tail -40 $O/r02s_memcheck.log
NB="python bench.py --config gnn --ops spmm --panel-rows 64 --dense-min 8 --steps 1 --warmup 1 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"spmm_dense|spmm_task" -c 2 -o $O/r02s_prof_gnn $NB > $O/r02s_ncu_gnn.log 2>&1; echo ncu $?

# round 2, session v: ncu of the phase-D TMA engine at 32-row panels on C4 (4 rows per consumer warp)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
O=gpurun_out
NB="python bench.py --config gnn --ops spmm --panel-rows 32 --dense-min 4 --steps 1 --warmup 1 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"spmm_dense" -c 1 -o $O/r02v_prof_gnn_p32 $NB > $O/r02v_ncu.log 2>&1; echo ncu $?

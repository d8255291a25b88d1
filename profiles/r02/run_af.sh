# round 2, session af: ncu of the SDDMM phase-D kernel (3-stage ring) on C5, 32-row panels, dense_min 4
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
O=gpurun_out
NB="python bench.py --config cf --ops sddmm --panel-rows 32 --dense-min 4 --steps 1 --warmup 1 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"sddmm_dense" -c 1 -o $O/r02af_prof_cf $NB > $O/r02af_ncu.log 2>&1; echo ncu $?

# round 2, session p: the TMA shared-memory phase-D engine at tall panels on C4 (GNN): reuse per
# staged column grows with the panel height (P=8: 2.5, P=16: 3.0)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
B="python bench.py --config gnn --ops spmm --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0"
for pd in "64 2" "64 4" "64 8" "128 2" "128 4" "32 2"; do set -- $pd
  timeout 900 $B --panel-rows $1 --dense-min $2 > $O/r02p_gnn_p$1_d$2.json 2> $O/r02p_gnn_p$1_d$2.err
done
B="python bench.py --config cf --ops sddmm --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0"
for pd in "64 2" "128 4"; do set -- $pd
  timeout 900 $B --panel-rows $1 --dense-min $2 > $O/r02p_cf_p$1_d$2.json 2> $O/r02p_cf_p$1_d$2.err
done

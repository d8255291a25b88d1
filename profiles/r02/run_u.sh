# round 2, session u: phase-D tiles at short panels now that every consumer warp has rows
# (rows per warp = panel/8): C4 SpMM, C5 SDDMM, C2 — against no-tile plans in the same call
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
O=gpurun_out
run() { cfg=$1; ops=$2; p=$3; d=$4; tag=$5
  timeout 900 python bench.py --config $cfg --ops $ops --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 \
    --extra-K none --panel-rows $p --dense-min $d --plan-cache /tmp/${cfg}_p${p}_d${d}.plan > $O/r02u_${cfg}_${tag}.json 2> $O/r02u_${cfg}_${tag}.err; }
run gnn spmm 64 64 notile_a
for pd in "16 2" "16 3" "16 4" "32 2" "32 3" "32 4" "32 6"; do set -- $pd; run gnn spmm $1 $2 p$1_d$2; done
run gnn spmm 64 64 notile_b
run cf sddmm 64 64 notile_a
for pd in "16 3" "32 3" "32 4"; do set -- $pd; run cf sddmm $1 $2 p$1_d$2; done
run cf sddmm 64 64 notile_b
run rmat spmm,sddmm 64 64 notile_a
for pd in "32 4" "32 8" "16 4"; do set -- $pd; run rmat spmm,sddmm $1 $2 p$1_d$2; done

# round 2, session ag: SDDMM phase-D consumers read staged rows only for groups holding an entry;
# 3-stage ring (adaptive) — parity, C5 and C4 tiled vs untiled
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m "gpu and not slow" -q -x 2>&1 | tail -2
run() { cfg=$1; ops=$2; p=$3; d=$4; tag=$5
  timeout 900 python bench.py --config $cfg --ops $ops --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 \
    --extra-K none --panel-rows $p --dense-min $d --plan-cache /tmp/${cfg}_p${p}_d${d}.plan > $O/r02ag_${cfg}_${tag}.json 2> $O/r02ag_${cfg}_${tag}.err; }
run cf sddmm 64 64 notile_a
run cf sddmm 32 4 p32_d4
run cf sddmm 32 6 p32_d6
run cf sddmm 16 4 p16_d4
run cf sddmm 32 3 p32_d3
run cf sddmm 64 64 notile_b
run gnn spmm,sddmm 32 4 both
run gnn spmm,sddmm 64 64 both_notile
NB="python bench.py --config cf --ops sddmm --panel-rows 32 --dense-min 4 --steps 1 --warmup 1 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none --plan-cache /tmp/cf_p32_d4.plan"
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"sddmm_dense" -c 1 -o $O/r02ag_prof_cf $NB > $O/r02ag_ncu.log 2>&1; echo ncu $?

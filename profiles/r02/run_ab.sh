# round 2, session ab: SDDMM phase-D consumer skips batch steps past a row's last entry — parity,
# C5 (CF SDDMM) tiled vs untiled
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m "gpu and not slow" -q -x 2>&1 | tail -3 > $O/r02ab_pt.log
cat $O/r02ab_pt.log
run() { cfg=$1; ops=$2; p=$3; d=$4; tag=$5
  timeout 900 python bench.py --config $cfg --ops $ops --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 \
    --extra-K none --panel-rows $p --dense-min $d --plan-cache /tmp/${cfg}_p${p}_d${d}.plan > $O/r02ab_${cfg}_${tag}.json 2> $O/r02ab_${cfg}_${tag}.err; }
run cf sddmm 64 64 notile_a
run cf sddmm 32 4 p32_d4
run cf sddmm 32 3 p32_d3
run cf sddmm 16 3 p16_d3
run cf sddmm 64 8 p64_d8
run cf sddmm 32 6 p32_d6
run cf sddmm 64 64 notile_b
run gnn spmm,sddmm 32 4 p32_d4_both
run gnn spmm,sddmm 64 64 notile_both

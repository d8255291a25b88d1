# round 2, session ae: SDDMM phase-D consumers read their X rows from shared memory (staged once
# per unit); ring depth 3 when it fits beside them, else 2
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m "gpu and not slow" -q -x 2>&1 | tail -2
run() { cfg=$1; ops=$2; p=$3; d=$4; tag=$5
  timeout 900 python bench.py --config $cfg --ops $ops --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 \
    --extra-K none --panel-rows $p --dense-min $d --plan-cache /tmp/${cfg}_p${p}_d${d}.plan > $O/r02ae_${cfg}_${tag}.json 2> $O/r02ae_${cfg}_${tag}.err; }
run cf sddmm 64 64 notile
run cf sddmm 32 4 p32_d4
run cf sddmm 32 6 p32_d6
run cf sddmm 64 8 p64_d8
run cf sddmm 16 4 p16_d4
run gnn spmm,sddmm 32 4 both

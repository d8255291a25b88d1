# round 2, session w: 16 consumer warps in the phase-D engine (default) and rows per warp by panel
# height — GPU parity (fast set), C2 bench, C4 / C5 tiled vs untiled plans
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m "gpu and not slow" -q -x 2>&1 | tail -3 > $O/r02w_pt.log
timeout 900 python bench.py --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --plan-cache /tmp/c2.plan > $O/r02w_bench.json 2> $O/r02w_bench.err
run() { cfg=$1; ops=$2; p=$3; d=$4; tag=$5
  timeout 900 python bench.py --config $cfg --ops $ops --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 \
    --extra-K none --panel-rows $p --dense-min $d --plan-cache /tmp/${cfg}_p${p}_d${d}.plan > $O/r02w_${cfg}_${tag}.json 2> $O/r02w_${cfg}_${tag}.err; }
run gnn spmm 64 64 notile_a
run gnn spmm 32 4 p32_d4
run gnn spmm 64 8 p64_d8
run gnn spmm 64 64 notile_b
run gnn spmm 32 4 p32_d4b
cat $O/r02w_pt.log

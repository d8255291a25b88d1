# round 2, session aa: phase-D units of up to 32 tiles (whole C4 panels: no split partials),
# column ids from global, one fence per split unit — parity, C4 tiled vs untiled, C2 bench
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
O=gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -m "gpu and not slow" -q -x 2>&1 | tail -3 > $O/r02aa_pt.log
cat $O/r02aa_pt.log
run() { cfg=$1; ops=$2; p=$3; d=$4; tag=$5
  timeout 900 python bench.py --config $cfg --ops $ops --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 \
    --extra-K none --panel-rows $p --dense-min $d --plan-cache /tmp/${cfg}_p${p}_d${d}.plan > $O/r02aa_${cfg}_${tag}.json 2> $O/r02aa_${cfg}_${tag}.err; }
run gnn spmm 64 64 notile_a
run gnn spmm 32 4 p32_d4
run gnn spmm 64 8 p64_d8
run gnn spmm 32 3 p32_d3
run gnn spmm 64 64 notile_b
run gnn spmm 32 4 p32_d4b
run cf sddmm 32 4 p32_d4
run cf sddmm 64 64 notile
timeout 900 python bench.py --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 > $O/r02aa_bench.json 2> $O/r02aa_bench.err

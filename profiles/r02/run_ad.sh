# round 2, session ad: SDDMM phase-D ring depth 2 vs 3 (the smaller unit blobs leave room for 3)
set -x
O=gpurun_out
run() { cfg=$1; ops=$2; p=$3; d=$4; tag=$5
  timeout 900 python bench.py --config $cfg --ops $ops --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 \
    --extra-K none --panel-rows $p --dense-min $d --plan-cache /tmp/${cfg}_p${p}_d${d}.plan > $O/r02ad_${cfg}_${tag}.json 2> $O/r02ad_${cfg}_${tag}.err; }
for st in 2 3; do
  SR_NVCC_DEFS="-DSR_SDDMM_STAGES=$st" python -c "from paper_conf_ppopp_jiangha20_b200 import _build; _build.build()" 2>&1 | tail -1
  [ $st = 3 ] && timeout 900 python -m pytest tests/test_gpu_parity.py -m "gpu and not slow" -q -x 2>&1 | tail -2
  run cf sddmm 32 4 s${st}_p32_d4
  run cf sddmm 32 6 s${st}_p32_d6
  run gnn spmm,sddmm 32 4 s${st}_both
done
run cf sddmm 64 64 notile
python -c "from paper_conf_ppopp_jiangha20_b200 import _build; _build.build()" 2>&1 | tail -1

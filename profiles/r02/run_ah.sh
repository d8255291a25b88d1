# round 2, session ah: SDDMM phase-D entry slots per group U = 1 / 2 / 4 (C5, C4)
set -x
O=gpurun_out
run() { cfg=$1; ops=$2; p=$3; d=$4; tag=$5
  timeout 900 python bench.py --config $cfg --ops $ops --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 \
    --extra-K none --panel-rows $p --dense-min $d --plan-cache /tmp/${cfg}_p${p}_d${d}.plan > $O/r02ah_${cfg}_${tag}.json 2> $O/r02ah_${cfg}_${tag}.err; }
for u in 1 2 4; do
  SR_NVCC_DEFS="-DSR_SDDMM_DENSE_U=$u" python -c "from paper_conf_ppopp_jiangha20_b200 import _build; _build.build()" 2>&1 | tail -1
  [ $u = 2 ] && timeout 900 python -m pytest tests/test_gpu_parity.py -m "gpu and not slow" -q -x 2>&1 | tail -2
  run cf sddmm 32 4 u${u}_p32_d4
  run cf sddmm 32 6 u${u}_p32_d6
  run gnn sddmm 32 4 u${u}_gnn
done
run cf sddmm 64 64 notile
run gnn sddmm 64 64 gnn_notile

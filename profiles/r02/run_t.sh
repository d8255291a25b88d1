# round 2, session t: phase-D TMA engine occupancy on C4 (GNN, 64-row panels): consumer warps per
# CTA (8 vs 16), CTAs per SM / stages (2 x 3 vs 3 x 2); rows per warp now 2/4/8/16 by panel height
set -x
O=gpurun_out
B="python bench.py --config gnn --ops spmm --steps 10 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0"
for v in "base:" "w16:-DSR_DENSE_WARPS=16" "c3s2:-DSR_DENSE_CTAS=3 -DSR_SPMM_STAGES=2"; do
  tag=${v%%:*}; defs=${v#*:}
  SR_NVCC_DEFS="$defs" python -c "from paper_conf_ppopp_jiangha20_b200 import _build; _build.build(force=True)" 2>&1 | tail -1
  for pd in "64 8" "64 4" "32 4"; do set -- $pd
    timeout 900 $B --panel-rows $1 --dense-min $2 --plan-cache /tmp/gnn_p$1_d$2.plan > $O/r02t_${tag}_p$1_d$2.json 2> $O/r02t_${tag}_p$1_d$2.err
  done
done
timeout 900 $B --plan-cache /tmp/gnn_default.plan > $O/r02t_notile.json 2> $O/r02t_notile.err
python -c "from paper_conf_ppopp_jiangha20_b200 import _build; _build.build(force=True)" 2>&1 | tail -1

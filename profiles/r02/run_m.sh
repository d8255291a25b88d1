# round 2, session m: L2 prefetch of the next entry batch's rows through the bulk-copy unit (SR_L2PF)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
SR_L2PF=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "k_sweep or long_rows or tiny or strided or set_values" 2>&1 | tail -2 > $O/r02m_pt_pf.log
B="python bench.py --steps 20 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --plan-cache /tmp/c2.plan"
for v in 0 1 0 1; do SR_L2PF=$v timeout 900 $B > $O/r02m_pf${v}_$RANDOM.json 2>/dev/null; done
M="dram__bytes_read.sum,lts__t_sector_hit_rate.pct,gpu__time_duration.sum,l1tex__data_pipe_lsu_wavefronts.sum,smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio"
NB="python bench.py --steps 1 --warmup 1 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none --plan-cache /tmp/c2.plan"
SR_L2PF=1 timeout 600 ncu --metrics $M --clock-control none -k regex:task -c 4 --csv $NB > $O/r02m_ncu_pf1.csv 2>/dev/null
tail -1 $O/r02m_pt_pf.log

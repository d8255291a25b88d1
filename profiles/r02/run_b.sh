# round 2, session b: phase-S kernel variants (SR_SPMM_S) and SDDMM column blocks (SR_SDDMM_COLBLOCKS)
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
O=gpurun_out
B="python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --plan-cache /tmp/c2.plan"
timeout 600 $B --ops spmm > $O/r02b_spmm_v0.json 2> $O/r02b_spmm_v0.err
for v in 1 2 3 4; do SR_SPMM_S=$v timeout 600 $B --ops spmm > $O/r02b_spmm_v$v.json 2> $O/r02b_spmm_v$v.err; done
for cb in 1 2 4 8; do SR_SDDMM_COLBLOCKS=$cb timeout 600 $B --ops sddmm > $O/r02b_sddmm_cb$cb.json 2> $O/r02b_sddmm_cb$cb.err; done
M="l1tex__data_pipe_lsu_wavefronts.sum,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,sm__warps_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum,l1tex__throughput.avg.pct_of_peak_sustained_elapsed,lts__throughput.avg.pct_of_peak_sustained_elapsed,launch__registers_per_thread"
NB="python bench.py --steps 1 --warmup 1 --min-warm-s 0 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --plan-cache /tmp/c2.plan"
for v in 0 1 3; do SR_SPMM_S=$v timeout 600 ncu --metrics $M --clock-control none -k regex:task -c 6 --csv $NB --ops spmm > $O/r02b_ncu_spmm_v$v.csv 2>/dev/null; done
for cb in 1 4; do SR_SDDMM_COLBLOCKS=$cb timeout 600 ncu --metrics $M --clock-control none -k regex:task -c 3 --csv $NB --ops sddmm --extra-K "" > $O/r02b_ncu_sddmm_cb$cb.csv 2>/dev/null; done
for v in 1 3 4; do SR_SPMM_S=$v timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "k_sweep or tile_widths or long_rows or tiny" 2>&1 | tail -2 > $O/r02b_pt_spmm$v.log; done
SR_SDDMM_COLBLOCKS=4 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "k_sweep or tile_widths or long_rows or tiny or set_values or shard" 2>&1 | tail -2 > $O/r02b_pt_cb4.log
tail -n1 $O/r02b_pt_*.log

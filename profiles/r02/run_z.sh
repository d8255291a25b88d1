# round 2, session z: reorder preprocessing of C2 with the Alg 3 live-pop masks and J=0 prefetches
set -x
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
O=gpurun_out
for i in 1 2; do
  timeout 900 python bench.py --steps 5 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none > $O/r02z_pre$i.json 2> $O/r02z_pre$i.err
done
SR_DEBUG_REORDER=1 SR_DEBUG_CLUSTER=1 timeout 900 python bench.py --steps 5 --no-cpu-baseline --no-oracle-reorder --e2e-steps 0 --extra-K none > $O/r02z_dbg.json 2> $O/r02z_dbg.err
grep -h "sr_reorder\|J>0\|cluster_rows" $O/r02z_dbg.err

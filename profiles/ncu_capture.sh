#!/bin/bash
# Usage (under gpurun): bash profiles/ncu_capture.sh <tag> <kernel-regex> <count> [bench args...]
# Captures `ncu --set full` of the first <count> launches matching <kernel-regex> in a short
# bench.py run, then exports text summaries into gpurun_out/ (the .ncu-rep is too large to
# bring back) and deletes the report.
tag=$1; kre=$2; cnt=$3; shift 3
mkdir -p gpurun_out
ncu --set full --clock-control none --import-source on -k regex:"$kre" -c "$cnt" -f -o /tmp/prof_$tag \
    python bench.py --steps 1 --warmup 1 --min-warm-s 0 --e2e-steps 0 --no-cpu-baseline "$@" > gpurun_out/ncu_${tag}.log 2>&1
ncu -i /tmp/prof_$tag.ncu-rep --page raw --csv > gpurun_out/ncu_${tag}_raw.csv 2>/dev/null
ncu -i /tmp/prof_$tag.ncu-rep --page details --csv > gpurun_out/ncu_${tag}_details.csv 2>/dev/null
ncu -i /tmp/prof_$tag.ncu-rep --page source --csv > gpurun_out/ncu_${tag}_source.csv 2>/dev/null
gzip -f gpurun_out/ncu_${tag}_source.csv
rm -f /tmp/prof_$tag.ncu-rep
ls -la gpurun_out/ | grep $tag

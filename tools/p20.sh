#!/bin/bash
# SASS-level profile of the search match kernel at a reduced reference count (fast ncu replays):
# full set + source page (per-instruction executed counts and stall samples) as CSV.
TAG=${1:-p20}; REFS=${2:-20000}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:match_kernel -s 1 -c 1 \
  -o gpurun_out/${TAG}_match python bench.py --steps 1 --warmup 3 --no-cpu-baseline --refs-per-gpu $REFS \
  > /dev/null 2> gpurun_out/${TAG}_full.err
ncu -i gpurun_out/${TAG}_match.ncu-rep --page source --csv --print-source sass > gpurun_out/${TAG}_sass.csv 2>/dev/null
ncu -i gpurun_out/${TAG}_match.ncu-rep --page raw --csv > gpurun_out/${TAG}_raw.csv 2>/dev/null
ls -la gpurun_out | grep ${TAG}

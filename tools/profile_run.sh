#!/bin/bash
# ncu evidence for the dominant kernel (run under gpurun; 1 GPU).
#   $1 = tag (file prefix), remaining args forwarded to bench.py
set -x
TAG=${1:-r1}; shift
mkdir -p gpurun_out
# launch list: every kernel with its device time (cold-cache, serialised)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline "$@" > gpurun_out/${TAG}_launches_bench.json 2> gpurun_out/${TAG}_launches_bench.err
# one full capture of the match kernel on a reduced reference count (same kernel, same launch config)
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:match_kernel -s 1 -c 1 \
  -o gpurun_out/${TAG}_match python bench.py --steps 1 --warmup 3 --no-cpu-baseline --refs-per-gpu 20000 "$@" \
  > gpurun_out/${TAG}_full_bench.json 2> gpurun_out/${TAG}_full_bench.err
ls -la gpurun_out

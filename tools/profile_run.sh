#!/bin/bash
# ncu evidence for the dominant kernel (run under gpurun; 1 GPU).  $1 = tag; rest -> bench.py
TAG=${1:-r1}; shift
mkdir -p gpurun_out
# 1) bench line (not under a profiler)
timeout 900 python bench.py "$@" > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
# 2) launch list: every kernel with its device time (cold-cache, serialised: compare SHARES)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline "$@" > /dev/null 2> gpurun_out/${TAG}_launches.err
# 3) one full capture of the match kernel at the bench configuration (first timed-path launch)
timeout 1800 ncu --set full --clock-control none --import-source on -k regex:match_kernel -s 1 -c 1 \
  -o gpurun_out/${TAG}_match python bench.py --steps 1 --warmup 3 --no-cpu-baseline "$@" \
  > /dev/null 2> gpurun_out/${TAG}_full.err
ls -la gpurun_out | grep ${TAG}

mkdir -p gpurun_out
TAG=${1:-p10}
timeout 300 python bench.py > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:match_kernel -s 1 -c 1 -o gpurun_out/${TAG}_match python tools/run_search.py 20000 256 1 > gpurun_out/${TAG}_ncu.log 2>&1

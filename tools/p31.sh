# f16 match kernel: pipe utilisations (one launch) + stall-sampled SASS
mkdir -p gpurun_out
timeout 600 ncu --set full --import-source on --clock-control none -k regex:match_f16 -c 1 -o gpurun_out/p31_f16 \
  python tools/bench_configs.py f16 > /dev/null 2> gpurun_out/p31.err
ncu -i gpurun_out/p31_f16.ncu-rep --page raw --csv > gpurun_out/p31_raw.csv 2>/dev/null
ncu -i gpurun_out/p31_f16.ncu-rep --page source --csv --print-source sass > gpurun_out/p31_sass.csv 2>/dev/null

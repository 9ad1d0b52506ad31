set -x
mkdir -p gpurun_out
python tools/run_search.py 20000 256 3 > gpurun_out/p1_run.txt 2>&1
TID_LIB=$PWD/paper_conf_icpp_wangzll21_b200/libtid_prof.so python tools/prof_epilogue.py 20000 > gpurun_out/p1_prof.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:match_kernel -s 1 -c 1 -o gpurun_out/p1_match python tools/run_search.py 20000 256 1 > gpurun_out/p1_ncu.log 2>&1
ls -la gpurun_out

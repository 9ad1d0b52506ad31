# A/B: GPU parity tests + C4-shard-sized search timing + prof buckets (1 GPU)
mkdir -p gpurun_out
TAG=${1:-p2}
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest.txt 2>&1
timeout 300 python tools/run_search.py 20000 256 3 > gpurun_out/${TAG}_run.txt 2>&1
TID_LIB=$PWD/paper_conf_icpp_wangzll21_b200/libtid_prof.so timeout 300 python tools/prof_epilogue.py 20000 > gpurun_out/${TAG}_prof.txt 2>&1

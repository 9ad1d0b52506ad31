mkdir -p gpurun_out
TAG=${1:-p8}
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/${TAG}_smoke.txt 2>&1 || { echo "smoke failed"; exit 1; }
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest.txt 2>&1
bash tools/ab.sh ${TAG} base
TID_LIB=$PWD/paper_conf_icpp_wangzll21_b200/libtid_prof.so timeout 300 python tools/prof_epilogue.py 20000 > gpurun_out/${TAG}_prof.txt 2>&1

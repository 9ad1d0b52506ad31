# A/B timing of library variants (TID_LIB) on one search configuration; $1 = tag, $2 = refs, rest = variant names
# (base = paper_conf_icpp_wangzll21_b200/libtid.so, X = libtid_X.so); each variant timed twice, interleaved
TAG=$1; R=$2; shift 2
mkdir -p gpurun_out
for rep in 1 2; do
for v in "$@"; do
  lib=$PWD/paper_conf_icpp_wangzll21_b200/libtid${v:+_$v}.so
  [ "$v" = "base" ] && lib=$PWD/paper_conf_icpp_wangzll21_b200/libtid.so
  echo "== $v" >> gpurun_out/${TAG}_ab.txt
  TID_LIB=$lib timeout 300 python tools/run_search.py $R 256 3 >> gpurun_out/${TAG}_ab.txt 2>&1
done
done

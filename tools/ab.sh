# A/B timing of library variants (TID_LIB) on a 20k-reference search; $1 = tag, rest = variant names
TAG=$1; shift
mkdir -p gpurun_out
for v in "$@"; do
  lib=$PWD/paper_conf_icpp_wangzll21_b200/libtid${v:+_$v}.so
  [ "$v" = "base" ] && lib=$PWD/paper_conf_icpp_wangzll21_b200/libtid.so
  echo "== $v" >> gpurun_out/${TAG}_ab.txt
  TID_LIB=$lib timeout 300 python tools/run_search.py 20000 256 3 >> gpurun_out/${TAG}_ab.txt 2>&1
done

# A/B of library variants at several (R, B) points: $1 = tag; $2 = "R:B R:B ..."; rest = variants
TAG=$1; PTS=$2; shift 2
for rep in 1 2; do for pt in $PTS; do for v in "$@"; do
  lib=$PWD/paper_conf_icpp_wangzll21_b200/libtid_$v.so; [ "$v" = "base" ] && lib=$PWD/paper_conf_icpp_wangzll21_b200/libtid.so
  echo "== $v ${pt}" >> gpurun_out/${TAG}_ab.txt
  TID_LIB=$lib timeout 300 python tools/run_search.py ${pt%%:*} ${pt##*:} 5 >> gpurun_out/${TAG}_ab.txt 2>&1
done; done; done

# A/B of the search epilogue scan modes (tid_tuning.scan 1 = two-partition, 2 = piece maxima + exact
# recompute) at several (R, B) points, interleaved, twice: $1 = tag; $2 = "R:B R:B ..."
TAG=$1; PTS=$2
for rep in 1 2; do for pt in $PTS; do for sc in 1 2; do
  echo "== scan=$sc ${pt}" >> gpurun_out/${TAG}_ab.txt
  TID_SCAN=$sc timeout 300 python tools/run_search.py ${pt%%:*} ${pt##*:} 5 >> gpurun_out/${TAG}_ab.txt 2>&1
done; done; done

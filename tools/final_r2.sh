# Round-2 evidence run (one B200, under gpurun): bench line, launch list, one ncu --set full capture of
# the match kernel at the bench configuration, secondary configurations with clocks, compute-sanitizer.
TAG=${1:-r2z}
mkdir -p gpurun_out
bash tools/profile_run.sh $TAG
python tools/summarize_profile.py $TAG > gpurun_out/${TAG}_summary.txt 2>&1
timeout 1500 python tools/bench_configs.py c1 c3 c2 sweep f16 table7 > gpurun_out/${TAG}_configs.jsonl 2> gpurun_out/${TAG}_configs.err
for t in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $t --print-limit 20 python tools/sanitize_run.py > gpurun_out/${TAG}_san_$t.txt 2>&1
done
ls -la gpurun_out | grep $TAG

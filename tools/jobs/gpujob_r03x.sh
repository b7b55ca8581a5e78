cd $GRAFT_REPO_ROOT
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_tiny.py > gpurun_out/r03x_sanitizer_$tool.log 2>&1
  echo "$tool rc=$? $(grep 'ERROR SUMMARY\|RACECHECK SUMMARY' gpurun_out/r03x_sanitizer_$tool.log | tail -2)"
done
SONG_BENCH_BACKEND=gloo timeout 900 python bench.py --gpus 2 --steps 10 --warmup 3 --no-parity --no-cpu-baseline > gpurun_out/r03x_bench_gpus2.log 2>&1; echo gpus2 $?; tail -1 gpurun_out/r03x_bench_gpus2.log | cut -c1-300

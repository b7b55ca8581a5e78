cd $GRAFT_REPO_ROOT
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r03av_gputests.log 2>&1; tail -1 gpurun_out/r03av_gputests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r03av_smoke.log 2>&1; tail -1 gpurun_out/r03av_smoke.log
timeout 1200 python bench.py --config glove200 --steps 10 --warmup 3 --cpu-seconds 5 --cpu-single-seconds 3 > gpurun_out/r03av_bench_glove200.log 2>&1
echo $(grep -o '"value": [0-9.]*' gpurun_out/r03av_bench_glove200.log | head -2) $(grep -o '"frac": [0-9.]*' gpurun_out/r03av_bench_glove200.log | head -1) $(grep -o '"ok": [a-z]*' gpurun_out/r03av_bench_glove200.log | tail -1)

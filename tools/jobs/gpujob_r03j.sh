cd $GRAFT_REPO_ROOT
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r03j_gputests.log 2>&1; tail -2 gpurun_out/r03j_gputests.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r03j_bench_sift1m.log 2>&1
timeout 1200 python bench.py --config nytimes256 --steps 20 --warmup 5 --cpu-seconds 5 --cpu-single-seconds 3 > gpurun_out/r03j_bench_nytimes256.log 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r03j_smoke.log 2>&1; tail -1 gpurun_out/r03j_smoke.log
for f in gpurun_out/r03j_bench_*.log; do echo $f $(grep -o '"value": [0-9.]*' $f | head -2) $(grep -o '"queue_len": [0-9]*' $f | head -1) $(grep -o '"ok": [a-z]*' $f | tail -1); done

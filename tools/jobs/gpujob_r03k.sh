cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "pipelined or host_and_device" > gpurun_out/r03k_gputests.log 2>&1; tail -2 gpurun_out/r03k_gputests.log
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r03k_bench_sift1m.log 2>&1
timeout 900 python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-parity > gpurun_out/r03k_bench_sift1m_50.log 2>&1
for f in gpurun_out/r03k_bench_*.log; do echo $f $(grep -o '"value": [0-9.]*' $f | head -3) $(grep -o '"host_results_match_device": [a-z]*' $f); done

cd $GRAFT_REPO_ROOT
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r03bi_gputests.log 2>&1; tail -1 gpurun_out/r03bi_gputests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r03bi_smoke.log 2>&1; tail -1 gpurun_out/r03bi_smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r03bi_bench_sift1m.log 2>&1
timeout 900 python bench.py --K 100 --steps 20 --warmup 5 --cpu-seconds 5 --cpu-single-seconds 3 > gpurun_out/r03bi_bench_sift1m_K100.log 2>&1
timeout 1200 python bench.py --config nytimes256 --steps 20 --warmup 5 --cpu-seconds 5 --cpu-single-seconds 3 > gpurun_out/r03bi_bench_nytimes256.log 2>&1
timeout 1200 python bench.py --config gist1m --steps 20 --warmup 5 --cpu-seconds 5 --cpu-single-seconds 3 > gpurun_out/r03bi_bench_gist1m.log 2>&1
timeout 1200 python bench.py --config glove200 --steps 10 --warmup 3 --cpu-seconds 5 --cpu-single-seconds 3 > gpurun_out/r03bi_bench_glove200.log 2>&1
for f in gpurun_out/r03bi_bench_*.log; do echo $f $(grep -o '"value": [0-9.]*' $f | head -2) $(grep -o '"queue_len": [0-9]*' $f | head -1) $(grep -o '"frac": [0-9.]*' $f | head -1) $(grep -o '"ok": [a-z]*' $f | tail -1); done
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/r03bi_reference.log 2>&1; echo ref $(grep -o "\"value\": [0-9.]*" gpurun_out/r03bi_reference.log | head -1)

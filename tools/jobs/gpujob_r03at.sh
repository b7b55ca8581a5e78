cd $GRAFT_REPO_ROOT
timeout 1200 python bench.py --config gist1m --steps 20 --warmup 5 --cpu-seconds 5 --cpu-single-seconds 3 > gpurun_out/r03at_bench_gist1m.log 2>&1

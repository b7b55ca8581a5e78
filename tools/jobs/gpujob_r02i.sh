set -x
cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/r02i_gputests.log 2>&1
tail -3 gpurun_out/r02i_gputests.log
timeout 900 python bench.py --config glove200 --queue-len 1280 --steps 5 --warmup 3 --cpu-seconds 3 --cpu-single-seconds 2 > gpurun_out/r02i_bench_glove200.log 2>&1
timeout 900 python bench.py --config nytimes256 --queue-len 144 --steps 10 --warmup 3 --cpu-seconds 3 --cpu-single-seconds 2 > gpurun_out/r02i_bench_nytimes256.log 2>&1
timeout 900 python tools/fig10_split.py --config glove200 --queue-lens 500,1280 --out gpurun_out/r02i_fig10_glove200.json > gpurun_out/r02i_fig10_glove200.log 2>&1
timeout 900 python bench.py --config glove200 --queue-len 1280 --queue-kind separate --steps 5 --warmup 3 --no-parity --no-cpu-baseline > gpurun_out/r02i_bench_glove200_sep.log 2>&1

cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests -q -m gpu -k "merge_graph_rows" > gpurun_out/r02x_gputests.log 2>&1
tail -2 gpurun_out/r02x_gputests.log
timeout 900 python -m pytest tests -q -m gpu -k "full_size_sampled_parity and glove" >> gpurun_out/r02x_gputests.log 2>&1
tail -2 gpurun_out/r02x_gputests.log
timeout 1200 python bench.py --config glove200 --steps 10 --warmup 3 --cpu-seconds 5 --cpu-single-seconds 3 > gpurun_out/r02x_bench_glove200.log 2>&1
grep "operating point" gpurun_out/r02x_bench_glove200.log

cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -q -m gpu -k "merge_graph_rows or full_size_sampled_parity" > gpurun_out/r02v_gputests.log 2>&1
tail -3 gpurun_out/r02v_gputests.log
timeout 1200 python bench.py --config glove200 --steps 10 --warmup 3 --cpu-seconds 5 --cpu-single-seconds 3 > gpurun_out/r02v_bench_glove200.log 2>&1
tail -c 1500 gpurun_out/r02v_bench_glove200.log

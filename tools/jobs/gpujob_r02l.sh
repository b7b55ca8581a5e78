cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -q -m gpu -k "sharding or peer or union or merge" > gpurun_out/r02l_gputests.log 2>&1
tail -3 gpurun_out/r02l_gputests.log
timeout 600 python bench.py --mode dataset --queue-len 28 --steps 10 --warmup 3 > gpurun_out/r02l_bench_dataset.log 2>&1
tail -c 800 gpurun_out/r02l_bench_dataset.log
for qk in auto union; do
timeout 600 python bench.py --K 100 --queue-len 100 --queue-kind $qk --steps 10 --warmup 3 --no-parity --no-cpu-baseline --cache /tmp/w_sift.pt > gpurun_out/r02l_bench_k100_$qk.log 2>&1
timeout 600 python bench.py --queue-len 28 --queue-kind $qk --steps 10 --warmup 3 --no-parity --no-cpu-baseline --cache /tmp/w_sift.pt > gpurun_out/r02l_bench_k10_$qk.log 2>&1
echo "$qk K100 $(grep -o '"value": [0-9.]*' gpurun_out/r02l_bench_k100_$qk.log | head -1) K10 $(grep -o '"value": [0-9.]*' gpurun_out/r02l_bench_k10_$qk.log | head -1)"
done

cd $GRAFT_REPO_ROOT
for sc in auto batch auto batch; do
  timeout 600 python bench.py --queue-len 20 --schedule $sc --steps 20 --warmup 5 --no-parity --no-cpu-baseline --cache /tmp/w_sift.pt > gpurun_out/r02sched_$sc.log 2>&1
  echo "$sc $(grep -o '"value": [0-9.]*' gpurun_out/r02sched_$sc.log | head -2 | tr '\n' ' ')"
done

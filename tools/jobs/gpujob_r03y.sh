cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests/test_gpu_multiquery.py -q -m gpu > gpurun_out/r03y_gputests_mq.log 2>&1; tail -3 gpurun_out/r03y_gputests_mq.log
# Fig. 8 on B200: queries per warp 1 / 2 / 4 in the packing kernel vs the production kernel
run() { timeout 900 python bench.py $1 --steps 10 --warmup 3 --no-cpu-baseline --cache /tmp/f8_sift.pt > gpurun_out/r03y_fig8_$2.log 2>&1; tail -1 gpurun_out/r03y_fig8_$2.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$2', d['value'], d['ms_per_step'], d['roofline']['n_dist'], d['roofline']['frac'], d['roofline']['kernel'], d['parity']['ok'] if 'parity' in d else '')"; }
for L in 16 64; do
  run "--queue-len $L" prod_L$L
  run "--queue-len $L --visited-cap -1 --queue-kind separate" prod_eager_L$L
  for G in 1 2 4; do run "--queue-len $L --visited-cap -1 --queries-per-warp $G" mq${G}_L$L; done
done

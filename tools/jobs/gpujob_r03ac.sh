cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_c_example.py tests/test_gpu_parity.py -q -m gpu -x -k "c_example or cuckoo or union or edges or bit_exact" > gpurun_out/r03ac_gputests.log 2>&1; tail -2 gpurun_out/r03ac_gputests.log
run() { SONG_LIB=paper_conf_icde_zhaotl20_b200/$1 timeout 600 python bench.py $2 --steps 20 --warmup 5 --no-parity --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', '$3', d['value'], d['ms_per_step'], d['roofline']['n_dist'], d['roofline']['frac'])"; }
run libsong.so "--queue-len 16 --cache /tmp/ab_sift.pt" warm > /dev/null
run libsong.so "--config glove200 --queue-len 160 --cache /tmp/ab_glove.pt" warm > /dev/null
for rep in 1 2; do
for lib in libsong.so libsong_prev.so; do
  run $lib "--queue-len 16 --cache /tmp/ab_sift.pt" L16
  run $lib "--config glove200 --queue-len 160 --cache /tmp/ab_glove.pt" G160
done
done

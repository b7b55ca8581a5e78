cd $GRAFT_REPO_ROOT
SONG_LIB=paper_conf_icde_zhaotl20_b200/libsong_slot.so timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -x -k "union or edges or bit_exact or toy or pipelined" > gpurun_out/r03be_gputests_slot.log 2>&1; tail -1 gpurun_out/r03be_gputests_slot.log
run() { SONG_LIB=paper_conf_icde_zhaotl20_b200/$1 timeout 600 python bench.py $2 --steps 20 --warmup 5 --no-parity --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', '$3', d['value'], d['ms_per_step'], d['roofline']['n_dist'], d['roofline']['frac'])"; }
run libsong.so "--K 100 --queue-len 100 --cache /tmp/ab_k100.pt" warm > /dev/null
run libsong.so "--config nytimes256 --queue-len 56 --cache /tmp/ab_nyt.pt" warm > /dev/null
run libsong.so "--queue-len 16 --cache /tmp/ab_sift.pt" warm > /dev/null
for rep in 1 2; do
  for lib in libsong.so libsong_slot.so; do
    run $lib "--K 100 --queue-len 100 --cache /tmp/ab_k100.pt" K100
    run $lib "--config nytimes256 --queue-len 56 --cache /tmp/ab_nyt.pt" NYT56
    run $lib "--queue-len 16 --cache /tmp/ab_sift.pt" L16
  done
done

cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -m gpu -k "host or pipelined" > gpurun_out/r03z_gputests.log 2>&1; tail -2 gpurun_out/r03z_gputests.log
run() { SONG_LIB=paper_conf_icde_zhaotl20_b200/$1 timeout 600 python bench.py $2 --steps 20 --warmup 5 --no-parity --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); e=d['e2e']; print('$1', '$3', d['value'], e['value'], e['per_call']['value'], e['per_call']['ms_per_step'])"; }
run libsong.so "--queue-len 16 --cache /tmp/ab_sift.pt" warm > /dev/null
for rep in 1 2; do
for lib in libsong.so libsong_cc1.so; do
  run $lib "--queue-len 16 --cache /tmp/ab_sift.pt" L16
done
done

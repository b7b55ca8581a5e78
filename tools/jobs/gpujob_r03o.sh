cd $GRAFT_REPO_ROOT
run() { SONG_LIB=paper_conf_icde_zhaotl20_b200/$1 timeout 900 python bench.py $2 --steps 10 --warmup 3 --no-parity --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', '$3', d['value'], d['ms_per_step'], d['roofline']['n_dist'], d['roofline']['frac'], d['e2e']['value'])"; }
run libsong.so "--config gist1m --queue-len 24 --cache /tmp/ab_gist.pt" warm
for rep in 1 2; do
for lib in libsong_song_xwide_rows8.so libsong_song_xwide_rows16.so; do
  run $lib "--config gist1m --queue-len 24 --cache /tmp/ab_gist.pt" G24
  run $lib "--config gist1m --queue-len 48 --cache /tmp/ab_gist.pt" G48
done
done
SONG_LIB=paper_conf_icde_zhaotl20_b200/libsong_song_xwide_rows8.so timeout 900 python bench.py --config gist1m --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r03o_bench_gist1m_rows8.log 2>&1; tail -1 gpurun_out/r03o_bench_gist1m_rows8.log | cut -c1-600

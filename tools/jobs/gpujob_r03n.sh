cd $GRAFT_REPO_ROOT
# A/B: GIST-shaped rows staged per round (SONG_XWIDE_ROWS 2/4/8) and two stage buffers
run() { SONG_LIB=paper_conf_icde_zhaotl20_b200/$1 timeout 900 python bench.py $2 --steps 10 --warmup 3 --no-parity --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', '$3', d['value'], d['ms_per_step'], d['roofline']['n_dist'], d['roofline']['frac'], d['e2e']['value'])"; }
run libsong.so "--config gist1m --queue-len 24 --cache /tmp/ab_gist.pt" warm
for rep in 1 2; do
for lib in libsong.so libsong_song_xwide_rows2.so libsong_song_xwide_rows8.so libsong_song_stage_bufs2.so; do
  run $lib "--config gist1m --queue-len 24 --cache /tmp/ab_gist.pt" G24
done
done
run libsong_song_stage_bufs2.so "--queue-len 16 --cache /tmp/ab_sift.pt" L16
run libsong.so "--queue-len 16 --cache /tmp/ab_sift.pt" L16

cd $GRAFT_REPO_ROOT
run() { SONG_LIB=paper_conf_icde_zhaotl20_b200/$1 timeout 600 python bench.py $2 --steps 10 --warmup 3 --no-parity --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', '$3', d['value'], d['ms_per_step'], d['roofline']['n_dist'], d['roofline']['frac'])"; }
run libsong.so "--config glove200 --queue-len 160 --cache /tmp/ab_glove.pt" warm > /dev/null
run libsong.so "--config gist1m --queue-len 24 --cache /tmp/ab_gist.pt" warm > /dev/null
for rep in 1 2; do
  for lib in libsong.so libsong_noslot.so; do
    run $lib "--config glove200 --queue-len 160 --cache /tmp/ab_glove.pt" G160
    run $lib "--config gist1m --queue-len 24 --cache /tmp/ab_gist.pt" G24
  done
done

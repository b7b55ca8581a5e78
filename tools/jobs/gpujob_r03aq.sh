cd $GRAFT_REPO_ROOT
for lib in libsong.so libsong_pw4.so libsong_pw8.so libsong_pw16.so libsong_xw8.so; do
  SONG_LIB=paper_conf_icde_zhaotl20_b200/$lib timeout 900 python tools/bench_rp.py --config mnist8m --n 8090000 --builder batched --bits 128 --max-L 64 > gpurun_out/r03aq_mnist8m_$lib.log 2>&1
  echo $lib $(grep "original L=\(24\|32\|48\|64\)" gpurun_out/r03aq_mnist8m_$lib.log | sed 's/.*L=\([0-9]*\).*qps=\([0-9,]*\)/L\1:\2/' | tr '\n' ' ')
done
run() { SONG_LIB=paper_conf_icde_zhaotl20_b200/$1 timeout 600 python bench.py $2 --steps 10 --warmup 3 --no-parity --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', '$3', d['value'], d['ms_per_step'], d['roofline']['n_dist'], d['roofline']['frac'])"; }
run libsong.so "--config gist1m --queue-len 24 --cache /tmp/ab_gist.pt" warm > /dev/null
for rep in 1 2; do
  for lib in libsong.so libsong_pw4.so libsong_pw8.so libsong_pw16.so libsong_xw8.so; do run $lib "--config gist1m --queue-len 24 --cache /tmp/ab_gist.pt" G24; done
done

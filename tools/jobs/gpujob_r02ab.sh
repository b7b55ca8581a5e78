cd $GRAFT_REPO_ROOT
for lib in libsong.so libsong_team.so libsong_r4b2.so libsong.so; do
  SONG_LIB=paper_conf_icde_zhaotl20_b200/$lib timeout 600 python bench.py --queue-len 20 --steps 20 --warmup 5 --no-parity --no-cpu-baseline --cache /tmp/w_sift.pt > gpurun_out/r02ab_$lib.log 2>&1
  echo "$lib $(grep -o '"value": [0-9.]*' gpurun_out/r02ab_$lib.log | head -1)"
done

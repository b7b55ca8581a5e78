cd $GRAFT_REPO_ROOT
for lib in libsong.so libsong_uf4_1.so libsong_uf16_3.so; do
  for cfg in "nytimes256 144" "glove200 1280" "glove200 512"; do set -- $cfg
    SONG_LIB=paper_conf_icde_zhaotl20_b200/$lib timeout 600 python bench.py --config $1 --queue-len $2 --steps 10 --warmup 3 --no-parity --no-cpu-baseline --cache /tmp/w_$1.pt > gpurun_out/r02j_${lib}_$1_$2.log 2>&1
    echo "$lib $1 $2 $(grep -o '"value": [0-9.]*' gpurun_out/r02j_${lib}_$1_$2.log | head -1) $(grep -o '"n_dist": [0-9]*' gpurun_out/r02j_${lib}_$1_$2.log)"
  done
done

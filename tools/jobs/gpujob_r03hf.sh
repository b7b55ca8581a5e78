cd $GRAFT_REPO_ROOT
for lib in libsong.so libsong_hf4.so; do
  for cfg in "nytimes256 56" "sift1m 16" "glove200 160"; do set -- $cfg
    SONG_LIB=paper_conf_icde_zhaotl20_b200/$lib timeout 600 python bench.py --config $1 --queue-len $2 --steps 20 --warmup 5 --no-parity --no-cpu-baseline --cache /tmp/w_$1.pt > gpurun_out/r03hf_${lib}_$1.log 2>&1
    echo "$lib $1 $(grep -o '"value": [0-9.]*' gpurun_out/r03hf_${lib}_$1.log | head -1) $(grep -o '"n_dist": [0-9]*' gpurun_out/r03hf_${lib}_$1.log)"
  done
done

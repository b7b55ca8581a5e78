cd $GRAFT_REPO_ROOT
for cfg in "gist1m 24 0" "glove200 224 0" "nytimes256 80 0" "sift1m 100 100"; do set -- $cfg
  EXTRA="--config $1"; [ "$3" != "0" ] && EXTRA="$EXTRA --K $3"
  timeout 600 python bench.py $EXTRA --queue-len $2 --no-parity --no-cpu-baseline --cache /tmp/w_$1_$3.pt --profile --steps 1 --warmup 1 > gpurun_out/r02i_prep_$1_$3.log 2>&1
  timeout 900 ncu --nvtx --nvtx-include "song_timed/" --set full --clock-control none -k regex:song_search -c 1 -o gpurun_out/r02i_full_$1_$3 \
    python bench.py $EXTRA --queue-len $2 --no-parity --no-cpu-baseline --cache /tmp/w_$1_$3.pt --profile --steps 1 --warmup 1 > gpurun_out/r02i_full_$1_$3.log 2>&1
  python tools/ncu_summary.py gpurun_out/r02i_full_$1_$3.ncu-rep > gpurun_out/r02i_ncu_summary_$1_$3.txt 2>&1
  echo "== $1 L=$2 K=$3"; cat gpurun_out/r02i_ncu_summary_$1_$3.txt | head -6
done

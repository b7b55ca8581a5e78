#!/bin/bash
# One-GPU profiling recipe (B200_PROFILING.md): launch list + one full capture.
# usage: bash gpurun_profile.sh <tag> [bench args...]
TAG=$1; shift
ARGS="--queue-len 48 $@"
mkdir -p gpurun_out
timeout 300 python bench.py $ARGS --cache /tmp/song_w.pt --profile --steps 1 --warmup 1 > gpurun_out/${TAG}_prep.log 2>&1
timeout 600 ncu --nvtx --nvtx-include "song_timed/" --metrics gpu__time_duration.sum --clock-control none \
  --csv --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py $ARGS --cache /tmp/song_w.pt --profile --steps 5 --warmup 2 > gpurun_out/${TAG}_launch.log 2>&1
timeout 900 ncu --nvtx --nvtx-include "song_timed/" --set full --clock-control none --import-source on \
  -k regex:song_search -c 1 -o gpurun_out/${TAG}_full \
  python bench.py $ARGS --cache /tmp/song_w.pt --profile --steps 1 --warmup 1 > gpurun_out/${TAG}_full.log 2>&1
for f in gpurun_out/${TAG}_*.log; do tail -n 3 $f; done

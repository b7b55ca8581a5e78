#!/bin/bash
# A/B of libsong variants on the bench workload (same cached SIFT1M-shaped index).
# usage: bash tools/ab.sh <lib1> <lib2> ...   (paths relative to the repo)
python bench.py --queue-len 48 --steps 1 --warmup 1 --cache /tmp/sw.pt --no-cpu-baseline > /dev/null 2>&1
for rep in 1 2; do
for lib in "$@"; do
  SONG_LIB=$lib python bench.py --queue-len 48 --steps 20 --warmup 5 --cache /tmp/sw.pt --no-cpu-baseline 2>/dev/null \
   | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lib', d['value'], d['ms_per_step'], d['roofline']['n_dist'])"
done
done

#!/bin/bash
# A/B of libsong variants with extra bench args (same cached SIFT1M-shaped index).
# usage: ARGS="--K 100 --queue-len 128" bash tools/ab_args.sh <lib1> <lib2> ...
python bench.py --queue-len 48 --steps 1 --warmup 1 --cache /tmp/sw.pt --no-cpu-baseline > /dev/null 2>&1
for rep in 1 2; do
for lib in "$@"; do
  SONG_LIB=$lib python bench.py $ARGS --steps 20 --warmup 5 --cache /tmp/sw.pt --no-cpu-baseline 2>/dev/null \
   | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$lib', d['value'], d['ms_per_step'], d['roofline']['n_dist'], d['roofline']['frac'])"
done
done

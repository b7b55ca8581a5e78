# graph-builder parameter sweep (song_build_graph_batched) on the bench workload:
# the operating point (recall@10 >= 0.95) per (build queue_len, batch_shift, prefix)
CFG=${CFG:-sift1m}
for a in ${SWEEP:-"64 1 65536" "64 2 65536" "64 3 65536" "64 4 65536"}; do
  set -- $a
  r=$(timeout 300 python bench.py --config $CFG --sweep-only --build-queue-len $1 --build-shift $2 --build-prefix $3 2>&1 | grep -o "graph [0-9.]*s\|operating point.*" | tr '\n' ' ' | cut -c1-260)
  echo "L_b=$1 shift=$2 prefix=$3: $r"
done

python bench.py --queue-len 48 --steps 1 --warmup 1 --cache /tmp/sw.pt --no-cpu-baseline > /dev/null 2>&1
for cap in -1 128 256 384 512 640 768; do
  python bench.py --queue-len 48 --steps 10 --warmup 3 --cache /tmp/sw.pt --no-cpu-baseline --visited-cap $cap 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read()); print($cap, d['value'], d['roofline']['n_dist'], d['ms_per_step'])"
done

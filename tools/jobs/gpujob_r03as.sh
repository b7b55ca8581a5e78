cd $GRAFT_REPO_ROOT
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r03as_gputests.log 2>&1; tail -1 gpurun_out/r03as_gputests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r03as_smoke.log 2>&1; tail -1 gpurun_out/r03as_smoke.log
tag=gist1m
timeout 600 python bench.py --config gist1m --queue-len 24 --no-parity --no-cpu-baseline --cache /tmp/w_$tag.pt --profile --steps 1 --warmup 1 > gpurun_out/r03as_prep_$tag.log 2>&1
timeout 900 ncu --nvtx --nvtx-include "song_timed/" --set full --clock-control none -k regex:song_search -c 1 -o /tmp/r03as_full_$tag \
  python bench.py --config gist1m --queue-len 24 --no-parity --no-cpu-baseline --cache /tmp/w_$tag.pt --profile --steps 1 --warmup 1 > gpurun_out/r03as_full_$tag.log 2>&1
python tools/ncu_summary.py /tmp/r03as_full_$tag.ncu-rep > gpurun_out/r03as_ncu_summary_$tag.txt 2>&1
cat gpurun_out/r03as_ncu_summary_$tag.txt
timeout 3000 python tools/bench_rp.py --config mnist8m --n 8090000 --builder batched --bits 128 --max-L 256 --out gpurun_out/r03as_mnist8m.json > gpurun_out/r03as_mnist8m.log 2>&1; echo mnist8m rc=$?
grep "original L=\(32\|48\|64\)\|hash-128 L=128" gpurun_out/r03as_mnist8m.log

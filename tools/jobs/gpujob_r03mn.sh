cd $GRAFT_REPO_ROOT
free -g | head -2
timeout 3000 python tools/bench_rp.py --config mnist8m --n 8090000 --builder batched --bits 128 --max-L 256 --out gpurun_out/r03mn_mnist8m.json > gpurun_out/r03mn_mnist8m.log 2>&1; echo mnist8m rc=$?
tail -5 gpurun_out/r03mn_mnist8m.log

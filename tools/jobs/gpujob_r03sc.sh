cd $GRAFT_REPO_ROOT
timeout 2400 python tools/bench_scaleout.py --mix 64:1:24 --parity-sample 100 --out gpurun_out/r03sc_100m_mixed.json > gpurun_out/r03sc_100m_mixed.log 2>&1; echo rc=$?
tail -3 gpurun_out/r03sc_100m_mixed.log | cut -c1-700
timeout 900 python bench.py --mode dataset --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/r03sc_bench_dataset.log 2>&1; echo ds rc=$?; tail -1 gpurun_out/r03sc_bench_dataset.log | cut -c1-600

cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=memory.total --format=csv
timeout 2400 python tools/bench_scaleout.py --mix 64:1:24 --parity-sample 100 --out gpurun_out/r02scale_100m_mixed.json > gpurun_out/r02scale_100m_mixed.log 2>&1; echo rc=$?
tail -4 gpurun_out/r02scale_100m_mixed.log | cut -c1-1500

cd $GRAFT_REPO_ROOT
timeout 1200 python tools/fig11_batch.py --points 10:16,100:100 --out gpurun_out/r03bc_fig11.json > gpurun_out/r03bc_fig11.log 2>&1; echo fig11 $?
tail -3 gpurun_out/r03bc_fig11.log | cut -c1-800
timeout 1800 python tools/bench_knobs.py --config sift1m --steps-list 1,2 --out gpurun_out/r03bc_fig7_sift1m.json > gpurun_out/r03bc_fig7_sift1m.log 2>&1; echo fig7 $?
tail -3 gpurun_out/r03bc_fig7_sift1m.log | cut -c1-800

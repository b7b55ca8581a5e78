set -x
cd $GRAFT_REPO_ROOT
timeout 900 python tools/fig10_split.py --config glove200 --queue-lens 50,100,500,1000,1280 --out gpurun_out/r02c_fig10_glove200.json > gpurun_out/r02c_fig10_glove200.log 2>&1
timeout 900 python tools/fig10_split.py --config gist1m --queue-lens 50,100,500,1000 --out gpurun_out/r02c_fig10_gist1m.json > gpurun_out/r02c_fig10_gist1m.log 2>&1
timeout 600 python tools/fig10_split.py --config sift1m --queue-lens 28,64,128 --out gpurun_out/r02c_fig10_sift1m.json > gpurun_out/r02c_fig10_sift1m.log 2>&1

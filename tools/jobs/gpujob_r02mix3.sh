cd $GRAFT_REPO_ROOT
python tools/mix3_probe.py --config nytimes256 --a batched:cosine:128:2 --b batched:cosine:64:1 --c exact:cosine --takes 16/24,20/28,24/28 --L 56,64,72,80 --out gpurun_out/r02mix3_nyt.json 2>&1 | grep "^nytimes"
python tools/mix3_probe.py --config glove200 --a exact:ip --b batched:cosine:128:2 --c batched:cosine:64:1 --takes 8/20,8/24,6/20 --L 160,192,224 --out gpurun_out/r02mix3_glove.json 2>&1 | grep "^glove"
python tools/mix3_probe.py --config gist1m --a exact:l2 --b batched:l2:128:2 --c batched:l2:64:1 --takes 24/28,20/28 --L 16,20,24 --out gpurun_out/r02mix3_gist.json 2>&1 | grep "^gist"

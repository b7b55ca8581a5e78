cd $GRAFT_REPO_ROOT
python tools/mix_graph_probe.py --config glove200 --a exact:ip --b batched:cosine --take 8,6 --bq 256 --bs 3 --L 96,128,160,192,224 --out gpurun_out/r02ip2_a.json 2>&1 | grep "take"
python tools/mix_graph_probe.py --config glove200 --a exact:ip --b batched:l2 --take 8 --L 96,128,160,192,224 --out gpurun_out/r02ip2_b.json 2>&1 | grep "take"
python tools/mix_graph_probe.py --config glove200 --a batched:cosine --b exact:ip --take 24,26 --L 96,128,160,192,224 --out gpurun_out/r02ip2_c.json 2>&1 | grep "take"

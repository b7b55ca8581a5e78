cd $GRAFT_REPO_ROOT
python tools/mix_graph_probe.py --config sift1m --a batched:l2:128:2 --b batched:l2:64:1 --take 16,24 --L 16,20,24,28 --out gpurun_out/r02r16mix_a.json 2>&1 | grep "take"
python tools/mix_graph_probe.py --config sift1m --a batched:l2:128:2 --b batched:l2:256:3 --take 16,24 --L 16,20,24,28 --out gpurun_out/r02r16mix_b.json 2>&1 | grep "take"

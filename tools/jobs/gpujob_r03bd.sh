cd $GRAFT_REPO_ROOT
timeout 1200 python tools/fig10_split.py --config sift1m --queue-lens 16,100 --out gpurun_out/r03bd_fig10_sift1m.json > gpurun_out/r03bd_fig10_sift1m.log 2>&1; echo fig10 sift $?
timeout 1200 python tools/fig10_split.py --config gist1m --queue-lens 24,100 --out gpurun_out/r03bd_fig10_gist1m.json > gpurun_out/r03bd_fig10_gist1m.log 2>&1; echo fig10 gist $?
grep "^\[fig10\] {" gpurun_out/r03bd_fig10_*.log | python -c "
import sys, json
for line in sys.stdin:
    f, _, j = line.partition('[fig10] ')
    d = json.loads(j)
    print(f.split('/')[-1][:22], d['queue_len'], d['share_e2e'], d['share_kernel_paper_grouping'])"

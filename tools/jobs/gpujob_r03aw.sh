cd $GRAFT_REPO_ROOT
tag=glove200
timeout 600 python bench.py --config glove200 --queue-len 160 --no-parity --no-cpu-baseline --cache /tmp/w_$tag.pt --profile --steps 1 --warmup 1 > gpurun_out/r03aw_prep_$tag.log 2>&1
timeout 900 ncu --nvtx --nvtx-include "song_timed/" --set full --clock-control none -k regex:song_search -c 1 -o /tmp/r03aw_full_$tag \
  python bench.py --config glove200 --queue-len 160 --no-parity --no-cpu-baseline --cache /tmp/w_$tag.pt --profile --steps 1 --warmup 1 > gpurun_out/r03aw_full_$tag.log 2>&1
python tools/ncu_summary.py /tmp/r03aw_full_$tag.ncu-rep > gpurun_out/r03aw_ncu_summary_$tag.txt 2>&1
cat gpurun_out/r03aw_ncu_summary_$tag.txt

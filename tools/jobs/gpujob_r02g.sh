set -x
cd $GRAFT_REPO_ROOT
ARGS="--config glove200 --queue-len 1280 --no-parity --no-cpu-baseline"
timeout 600 python bench.py $ARGS --cache /tmp/song_glove.pt --profile --steps 1 --warmup 1 > gpurun_out/r02g_prep.log 2>&1
timeout 900 ncu --nvtx --nvtx-include "song_timed/" --set full --clock-control none --import-source on \
  -k regex:song_search -c 1 -o gpurun_out/r02g_glove_full \
  python bench.py $ARGS --cache /tmp/song_glove.pt --profile --steps 1 --warmup 1 > gpurun_out/r02g_full.log 2>&1
python tools/ncu_summary.py gpurun_out/r02g_glove_full.ncu-rep > gpurun_out/r02g_ncu_summary.txt 2>&1
python tools/sass_by_line.py gpurun_out/r02g_glove_full.ncu-rep paper_conf_icde_zhaotl20_b200/libsong.so song_search_kernelILi2ELi1ELi0ELi0ELb0 > gpurun_out/r02g_sass_by_line.txt 2>&1
tail -5 gpurun_out/r02g_full.log

cd $GRAFT_REPO_ROOT
bash tools/gpurun_profile.sh r03h --queue-len 16
python tools/ncu_summary.py gpurun_out/r03h_full.ncu-rep > gpurun_out/r03h_ncu_summary.txt 2>&1
python tools/launch_summary.py gpurun_out/r03h_launches.csv "ncu --metrics gpu__time_duration.sum --clock-control none, timed region of bench.py --queue-len 16 --steps 5 (r03h, R18 graph of 3)" > gpurun_out/r03h_launches_summary.txt 2>&1
python tools/sass_by_line.py gpurun_out/r03h_full.ncu-rep paper_conf_icde_zhaotl20_b200/libsong.so song_search_kernelILi1ELi0ELi0ELi1ELb0 > gpurun_out/r03h_sass_by_line.txt 2>&1
rm -f gpurun_out/r03h_full.ncu-rep
for cfg in "glove200 160" "nytimes256 56"; do set -- $cfg
  timeout 600 python bench.py --config $1 --queue-len $2 --no-parity --no-cpu-baseline --cache /tmp/w_$1.pt --profile --steps 1 --warmup 1 > gpurun_out/r03i_prep_$1.log 2>&1
  timeout 900 ncu --nvtx --nvtx-include "song_timed/" --set full --clock-control none -k regex:song_search -c 1 -o /tmp/r03i_full_$1 \
    python bench.py --config $1 --queue-len $2 --no-parity --no-cpu-baseline --cache /tmp/w_$1.pt --profile --steps 1 --warmup 1 > gpurun_out/r03i_full_$1.log 2>&1
  python tools/ncu_summary.py /tmp/r03i_full_$1.ncu-rep > gpurun_out/r03i_ncu_summary_$1.txt 2>&1
done
cat gpurun_out/r03h_ncu_summary.txt gpurun_out/r03h_launches_summary.txt gpurun_out/r03i_ncu_summary_*.txt

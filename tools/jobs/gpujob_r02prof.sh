cd $GRAFT_REPO_ROOT
bash tools/gpurun_profile.sh r02h --queue-len 20
python tools/ncu_summary.py gpurun_out/r02h_full.ncu-rep > gpurun_out/r02h_ncu_summary.txt 2>&1
python tools/launch_summary.py gpurun_out/r02h_launches.csv "ncu --metrics gpu__time_duration.sum --clock-control none, timed region of bench.py --queue-len 20 --steps 5 (r02h, R18 graph)" > gpurun_out/r02h_launches_summary.txt 2>&1
python tools/sass_by_line.py gpurun_out/r02h_full.ncu-rep paper_conf_icde_zhaotl20_b200/libsong.so song_search_kernelILi1ELi0ELi0ELi1ELb0 > gpurun_out/r02h_sass_by_line.txt 2>&1
cat gpurun_out/r02h_ncu_summary.txt gpurun_out/r02h_launches_summary.txt

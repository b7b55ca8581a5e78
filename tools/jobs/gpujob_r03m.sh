cd $GRAFT_REPO_ROOT
# K=100 operating point: launch list + ncu full capture + per-line SASS, and the in-kernel stage split
bash tools/gpurun_profile.sh r03m --K 100 --queue-len 100
python tools/ncu_summary.py gpurun_out/r03m_full.ncu-rep > gpurun_out/r03m_ncu_summary.txt 2>&1
python tools/launch_summary.py gpurun_out/r03m_launches.csv "ncu --metrics gpu__time_duration.sum --clock-control none, timed region of bench.py --K 100 --queue-len 100 --steps 5 (r03m, R16 graph)" > gpurun_out/r03m_launches_summary.txt 2>&1
python tools/sass_by_line.py gpurun_out/r03m_full.ncu-rep paper_conf_icde_zhaotl20_b200/libsong.so song_search_kernelILi1ELi0ELi0ELi4ELb0 > gpurun_out/r03m_sass_by_line.txt 2>&1
rm -f gpurun_out/r03m_full.ncu-rep
timeout 900 python tools/fig10_split.py --config sift1m --queue-lens 16,100 --out gpurun_out/r03m_fig10_sift1m.json > gpurun_out/r03m_fig10_sift1m.log 2>&1; echo fig10 $?
cat gpurun_out/r03m_ncu_summary.txt gpurun_out/r03m_launches_summary.txt; head -40 gpurun_out/r03m_sass_by_line.txt; tail -3 gpurun_out/r03m_fig10_sift1m.log

cd $GRAFT_REPO_ROOT
bash tools/gpurun_profile.sh r03ba --queue-len 16
python tools/ncu_summary.py gpurun_out/r03ba_full.ncu-rep > gpurun_out/r03ba_ncu_summary.txt 2>&1
python tools/launch_summary.py gpurun_out/r03ba_launches.csv "ncu --metrics gpu__time_duration.sum --clock-control none, timed region of bench.py --queue-len 16 --steps 5 (r03ba, R18 graph of 3, union W in registers)" > gpurun_out/r03ba_launches_summary.txt 2>&1
python tools/sass_by_line.py gpurun_out/r03ba_full.ncu-rep paper_conf_icde_zhaotl20_b200/libsong.so song_search_kernelILi1ELi0ELi0ELi9ELb0 > gpurun_out/r03ba_sass_by_line.txt 2>&1
rm -f gpurun_out/r03ba_full.ncu-rep
for cfg in "sift1m 100 --K_100" "nytimes256 56"; do set -- $cfg
  extra=$(echo "$3" | tr '_' ' ')
  tag=$1; [ -n "$3" ] && tag=${1}_K100
  timeout 600 python bench.py --config $1 --queue-len $2 $extra --no-parity --no-cpu-baseline --cache /tmp/w_$tag.pt --profile --steps 1 --warmup 1 > gpurun_out/r03ba_prep_$tag.log 2>&1
  timeout 900 ncu --nvtx --nvtx-include "song_timed/" --set full --clock-control none -k regex:song_search -c 1 -o /tmp/r03ba_full_$tag \
    python bench.py --config $1 --queue-len $2 $extra --no-parity --no-cpu-baseline --cache /tmp/w_$tag.pt --profile --steps 1 --warmup 1 > gpurun_out/r03ba_full_$tag.log 2>&1
  python tools/ncu_summary.py /tmp/r03ba_full_$tag.ncu-rep > gpurun_out/r03ba_ncu_summary_$tag.txt 2>&1
done
grep -h "kernel:\|duration\|dram__bytes\|warps_active\|issue_active" gpurun_out/r03ba_ncu_summary*.txt; cat gpurun_out/r03ba_launches_summary.txt

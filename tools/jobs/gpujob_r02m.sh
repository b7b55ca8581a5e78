cd $GRAFT_REPO_ROOT
for tool in memcheck racecheck synccheck initcheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_tiny.py > gpurun_out/r02m_sanitizer_$tool.log 2>&1
  echo "$tool rc=$? $(grep -c 'ERROR SUMMARY' gpurun_out/r02m_sanitizer_$tool.log) $(grep 'ERROR SUMMARY\|RACECHECK SUMMARY' gpurun_out/r02m_sanitizer_$tool.log | tail -2)"
done
timeout 1200 python tools/bench_knobs.py --config sift1m --steps-list 1 --out gpurun_out/r02m_fig7_sift1m.json > gpurun_out/r02m_fig7_sift1m.log 2>&1; echo fig7 $?
timeout 900 python tools/fig11_batch.py --out gpurun_out/r02m_fig11.json > gpurun_out/r02m_fig11.log 2>&1; echo fig11 $?
timeout 900 python tools/fig10_split.py --config gist1m --queue-lens 50,100,500,1000 --out gpurun_out/r02m_fig10_gist1m.json > gpurun_out/r02m_fig10_gist1m.log 2>&1; echo fig10g $?
timeout 900 python tools/fig10_split.py --config glove200 --queue-lens 50,100,500,1000,1280 --out gpurun_out/r02m_fig10_glove200.json > gpurun_out/r02m_fig10_glove200.log 2>&1; echo fig10 $?
timeout 2400 python tools/bench_rp.py --config mnist8m --n 8090000 --builder batched --bits 128 --max-L 256 --out gpurun_out/r02m_mnist8m.json > gpurun_out/r02m_mnist8m.log 2>&1; echo mnist8m $?

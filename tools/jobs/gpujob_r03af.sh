cd $GRAFT_REPO_ROOT
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r03af_gputests.log 2>&1; tail -2 gpurun_out/r03af_gputests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r03af_smoke.log 2>&1; tail -1 gpurun_out/r03af_smoke.log

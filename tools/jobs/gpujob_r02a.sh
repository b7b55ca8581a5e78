set -x
cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r02a_smoke.log 2>&1
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/r02a_gputests.log 2>&1
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/r02a_bench.log 2>&1
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/r02a_ref.log 2>&1
SONG_BENCH_BACKEND=gloo timeout 900 python bench.py --gpus 2 --steps 10 --warmup 3 --no-parity > gpurun_out/r02a_bench_gpus2.log 2>&1
tail -3 gpurun_out/r02a_gputests.log

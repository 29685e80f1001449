set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gputests.log 2>&1; echo tests=$?
timeout 300 python bench.py --steps 10 --warmup 3 > gpurun_out/bench.log 2>&1; echo bench=$?
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline --smem-split 1 > gpurun_out/bench_split.log 2>&1; echo bench=$?
tail -3 gpurun_out/gputests.log; tail -1 gpurun_out/bench.log; tail -1 gpurun_out/bench_split.log

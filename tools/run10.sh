python -m pytest tests -m gpu -x -q --timeout 900 > gpurun_out/t10.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t10.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ecoli10.json 2> gpurun_out/ecoli10.err
timeout 600 python bench.py --config chr14 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/chr14_10.json 2> gpurun_out/chr14_10.err
timeout 600 python bench.py --config tiny --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/tiny10.json 2> gpurun_out/tiny10.err

set -x
python -m pytest tests -m gpu -x -q --timeout 900 > gpurun_out/t2.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t2.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ecoli2.json 2> gpurun_out/ecoli2.err
timeout 900 python bench.py --config chr14 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/chr14_2.json 2> gpurun_out/chr14_2.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv --log-file gpurun_out/chr14_launches2.csv python bench.py --config chr14 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/chr14_ncu2.log 2>&1

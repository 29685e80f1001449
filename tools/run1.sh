set -x
python -m pytest tests -m gpu -x -q --timeout 900 > gpurun_out/t1.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t1.log
timeout 900 python bench.py --config chr14 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/chr14.json 2> gpurun_out/chr14.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/chr14_launches.csv python bench.py --config chr14 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/chr14_ncu.log 2>&1

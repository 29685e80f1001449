#!/bin/bash
# r02y: launch list (per-kernel times) of the chr14 step with the two-level counting-sort scatter,
# and an ncu source capture of its two levels
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "two_level" > gpurun_out/r02y_tests.log 2>&1; echo tests=$?; tail -1 gpurun_out/r02y_tests.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv --log-file gpurun_out/r02y_launches.csv \
  python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:'ts_level' -s 2 -c 2 -o gpurun_out/r02y_ts -f \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/r02y_ncu.log 2>&1; echo "ncu=$?"

#!/bin/bash
# round 2: GPU tests (except the long full-size ones), default bench (chr14), bumblebee bench
mkdir -p gpurun_out
python -m paper_conf_icdcs_qiul17_b200.build > gpurun_out/r02b_build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py -p no:randomly > gpurun_out/r02b_pytest.log 2>&1; echo rc=$? >> gpurun_out/r02b_pytest.log
timeout 900 python bench.py > gpurun_out/r02b_bench_chr14.json 2> gpurun_out/r02b_bench_chr14.err
timeout 900 python bench.py --config bumblebee --steps 5 --no-cpu-baseline > gpurun_out/r02b_bench_bbee.json 2> gpurun_out/r02b_bench_bbee.err

#!/bin/bash
# r02p: health check of the restored tree (GPU tests minus full-size, chr14 + bumblebee bench)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02p_pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/r02p_pytest.log
timeout 900 python bench.py --no-cpu-baseline --steps 10 --warmup 3 > gpurun_out/r02p_chr14.json 2> gpurun_out/r02p_chr14.err; echo bench=$?
python -c "import json; d=json.load(open('gpurun_out/r02p_chr14.json')); print(d['value']/1e9, d['breakdown_ms'], d['roofline']['frac'])"
timeout 900 python bench.py --no-cpu-baseline --steps 5 --warmup 3 --config bumblebee > gpurun_out/r02p_bbee.json 2> gpurun_out/r02p_bbee.err; echo bench=$?
python -c "import json; d=json.load(open('gpurun_out/r02p_bbee.json')); print(d['value']/1e9, d['breakdown_ms'], d['roofline']['frac'])"

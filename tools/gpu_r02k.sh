#!/bin/bash
# r02k: tests, bumblebee bench (compile-time K=63 MSP), f1 sweep on chr14, whole-human-shaped streaming run
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02k_pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/r02k_pytest.log
timeout 900 python bench.py --config bumblebee --no-cpu-baseline --steps 5 --warmup 3 > gpurun_out/r02k_bbee.json 2> gpurun_out/r02k_bbee.err
python -c "import json; d=json.load(open('gpurun_out/r02k_bbee.json')); print('bbee', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], round(d['roofline']['frac'],3))" || tail -3 gpurun_out/r02k_bbee.err
timeout 1500 python tools/f1_sweep.py > gpurun_out/r02k_f1_chr14.jsonl 2> gpurun_out/r02k_f1.err; echo f1=$?; wc -l gpurun_out/r02k_f1_chr14.jsonl
timeout 2400 python tools/human_run.py --scale 0.125 > gpurun_out/r02k_human.json 2> gpurun_out/r02k_human.err; echo human=$?; cat gpurun_out/r02k_human.json; tail -3 gpurun_out/r02k_human.err

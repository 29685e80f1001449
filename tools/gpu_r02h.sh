#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02h_pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/r02h_pytest.log
timeout 900 python bench.py --config bumblebee --no-cpu-baseline --steps 5 --warmup 3 > gpurun_out/r02h_bbee.json 2> gpurun_out/r02h_bbee.err
python -c "import json; d=json.load(open('gpurun_out/r02h_bbee.json')); print('bbee', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'])" || tail -3 gpurun_out/r02h_bbee.err
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:smem_subgraph -s 3 -c 1 -o gpurun_out/r02h_bbee_smem -f \
    python bench.py --config bumblebee --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r02h_ncu.log 2>&1; echo "ncu=$?"

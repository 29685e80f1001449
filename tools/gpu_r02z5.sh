#!/bin/bash
# r02z5: the committed state -- smoke, every GPU test but the full-size ones, bumblebee + chr14 bench lines
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r02z5_smoke.log 2>&1; echo smoke=$?; tail -1 gpurun_out/r02z5_smoke.log
timeout 1200 python -m pytest tests -m gpu -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02z5_pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/r02z5_pytest.log
timeout 900 python bench.py --config bumblebee --steps 5 --no-cpu-baseline > gpurun_out/r02z5_bench_bbee.json 2> gpurun_out/r02z5_bench_bbee.err; echo bbee=$?
timeout 900 python bench.py --no-cpu-baseline > gpurun_out/r02z5_bench_chr14.json 2> gpurun_out/r02z5_bench_chr14.err; echo chr14=$?
for f in bbee chr14; do python -c "import json; d=json.load(open('gpurun_out/r02z5_bench_$f.json')); print('$f', round(d['value']/1e9,3), round(d['ms_per_step'],3), d['breakdown_ms'], d['roofline']['frac'], d['roofline']['onchip']['stale'], d['gpu_launches'])"; done

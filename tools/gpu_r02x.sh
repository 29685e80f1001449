#!/bin/bash
# r02x: two-level counting-sort scatter (ts_level_a/b) -- parity (scatter tests, multi-GPU peers), then
# same-box A/B: one level vs two levels on chr14 (4-word records), bumblebee and E. coli
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "two_level or fine_pids or staging_overflow" > gpurun_out/r02x_scatter_tests.log 2>&1; echo scatter_tests=$?; tail -2 gpurun_out/r02x_scatter_tests.log
timeout 900 python -m pytest tests/test_gpu_multi.py -x -q > gpurun_out/r02x_multi.log 2>&1; echo multi=$?; tail -2 gpurun_out/r02x_multi.log
run() { tag=$1; shift; timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02x_$tag.json 2> gpurun_out/r02x_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02x_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], d['stats']['checksum'])" 2>/dev/null || tail -3 gpurun_out/r02x_$tag.err; }
run chr14_two --steps 10
run chr14_one --steps 10 --scatter one
run bbee_two --steps 5 --config bumblebee --scatter two
run bbee_one --steps 5 --config bumblebee
run ecoli_two --steps 10 --config ecoli --scatter two
run ecoli_one --steps 10 --config ecoli

#!/bin/bash
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
timeout 900 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02m_pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/r02m_pytest.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$V/$lib/libdbg.so timeout 900 python bench.py --no-cpu-baseline --steps 5 --warmup 3 "$@" > gpurun_out/r02m_$tag.json 2> gpurun_out/r02m_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02m_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], round(d['roofline']['frac'],3), d['config']['records'])" 2>/dev/null || tail -3 gpurun_out/r02m_$tag.err; }
run bbee_unroll unroll --config bumblebee
run bbee_gen gen --config bumblebee
timeout 900 compute-sanitizer --tool memcheck python tools/sanitize_driver.py > gpurun_out/r02m_memcheck.log 2>&1; echo memcheck=$?; tail -2 gpurun_out/r02m_memcheck.log

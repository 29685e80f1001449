#!/bin/bash
# r02w: 24-bit fine pid header + top-aligned reading-V minimizer: every GPU test but full-size; chr14 A/B vs HEAD~
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
timeout 1200 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02w_pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/r02w_pytest.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$lib timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02w_$tag.json 2> gpurun_out/r02w_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02w_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], d['stats']['checksum'])" 2>/dev/null || tail -3 gpurun_out/r02w_$tag.err; }
run chr14_new paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 10
run chr14_kold $V/kold/libdbg.so --steps 10
run chr14_new2 paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 10
run chr14_kold2 $V/kold/libdbg.so --steps 10

#!/bin/bash
# r02z6: two-level scatter bucket count (<= 1024 / 2048 (default) / 4096 buckets)
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
DBG_LIB_PATH=$V/b4096/libdbg.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "two_level" > gpurun_out/r02z6_tests.log 2>&1; echo tests=$?; tail -1 gpurun_out/r02z6_tests.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$lib timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02z6_$tag.json 2> gpurun_out/r02z6_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02z6_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'])" 2>/dev/null || tail -3 gpurun_out/r02z6_$tag.err; }
run chr14_b2048 paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 10
run chr14_b1024 $V/b1024/libdbg.so --steps 10
run chr14_b4096 $V/b4096/libdbg.so --steps 10
run bbee_b2048 paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 5 --config bumblebee
run bbee_b1024 $V/b1024/libdbg.so --steps 5 --config bumblebee
run bbee_b4096 $V/b4096/libdbg.so --steps 5 --config bumblebee

#!/bin/bash
# r02z4: warp-MSP occupancy (4 CTAs x 8 warps per SM, 192 descriptors) and 512-thread scatter tiles (2 CTAs/SM)
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
DBG_LIB_PATH=$V/w4/libdbg.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "warp_msp or ragged or long_reads" > gpurun_out/r02z4_tests_w4.log 2>&1; echo tests_w4=$?; tail -1 gpurun_out/r02z4_tests_w4.log
DBG_LIB_PATH=$V/ts512/libdbg.so timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "two_level" > gpurun_out/r02z4_tests_ts512.log 2>&1; echo tests_ts512=$?; tail -1 gpurun_out/r02z4_tests_ts512.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$lib timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02z4_$tag.json 2> gpurun_out/r02z4_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02z4_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], d['stats']['checksum'])" 2>/dev/null || tail -3 gpurun_out/r02z4_$tag.err; }
run bbee_base paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 5 --config bumblebee
run bbee_w4 $V/w4/libdbg.so --steps 5 --config bumblebee
run bbee_ts512 $V/ts512/libdbg.so --steps 5 --config bumblebee
run chr14_base paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 10
run chr14_ts512 $V/ts512/libdbg.so --steps 10

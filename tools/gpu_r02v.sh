#!/bin/bash
# r02v: warp-MSP edge-case test; two-slot probe (DBG_PROBE2) parity + A/B on bumblebee; full-size parity
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k warp_msp > gpurun_out/r02v_warptest.log 2>&1; echo "warptest=$?"; tail -1 gpurun_out/r02v_warptest.log
DBG_LIB_PATH=$V/probe2/libdbg.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r02v_pytest_probe2.log 2>&1; echo "pytest probe2=$?"; tail -1 gpurun_out/r02v_pytest_probe2.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$lib timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02v_$tag.json 2> gpurun_out/r02v_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02v_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], d['stats']['checksum'])" 2>/dev/null || tail -3 gpurun_out/r02v_$tag.err; }
run bbee_base paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 5 --config bumblebee
run bbee_probe2 $V/probe2/libdbg.so --steps 5 --config bumblebee
run bbee_base2 paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 5 --config bumblebee
run bbee_probe2b $V/probe2/libdbg.so --steps 5 --config bumblebee
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -x -q > gpurun_out/r02v_fullsize.log 2>&1; echo "fullsize=$?"; tail -2 gpurun_out/r02v_fullsize.log

#!/bin/bash
# r02q: warp-parallel MSP kernel -- parity, then same-box A/B against the thread-per-read kernels
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r02q_parity.log 2>&1; echo parity=$?; tail -3 gpurun_out/r02q_parity.log
timeout 600 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02q_pytest.log 2>&1; echo pytest=$?; tail -3 gpurun_out/r02q_pytest.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$lib timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02q_$tag.json 2> gpurun_out/r02q_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02q_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], d['stats']['checksum'])" 2>/dev/null || tail -3 gpurun_out/r02q_$tag.err; }
run chr14_warp paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 10
run chr14_thread $V/thread/libdbg.so --steps 10
run bbee_warp paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 5 --config bumblebee
run bbee_thread $V/thread/libdbg.so --steps 5 --config bumblebee
run ecoli_warp paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 10 --config ecoli
run ecoli_thread $V/thread/libdbg.so --steps 10 --config ecoli

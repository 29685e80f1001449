#!/bin/bash
# r02z3: TMA-staged counting-sort tiles (DBG_TS_TMA: one bulk copy per tile, permutation in shared memory,
# 2 CTAs/SM) vs the in-register tiles (8/4 records per thread); parity of both
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi.py -x -q -k "two_level or fine_pids or staging_overflow or sharded" > gpurun_out/r02z3_tests_reg.log 2>&1; echo tests_reg=$?; tail -1 gpurun_out/r02z3_tests_reg.log
DBG_LIB_PATH=$V/tma/libdbg.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "two_level or fine_pids or staging_overflow" > gpurun_out/r02z3_tests_tma.log 2>&1; echo tests_tma=$?; tail -1 gpurun_out/r02z3_tests_tma.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$lib timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02z3_$tag.json 2> gpurun_out/r02z3_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02z3_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], d['stats']['checksum'])" 2>/dev/null || tail -3 gpurun_out/r02z3_$tag.err; }
run chr14_reg paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 10
run chr14_tma $V/tma/libdbg.so --steps 10
run bbee_reg paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 5 --config bumblebee
run bbee_tma $V/tma/libdbg.so --steps 5 --config bumblebee

#!/bin/bash
# r02d: GPU tests on the new kernels, then A/B: two-level flat scatter vs one level vs per-bucket
# level 2 (chr14), chr14 fine_p 11 vs auto, bumblebee register-blocked MSP (K = 63) vs generic
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
timeout 1200 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02d_pytest.log 2>&1; echo pytest=$? >> gpurun_out/r02d_pytest.log; tail -3 gpurun_out/r02d_pytest.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$V/$lib/libdbg.so timeout 900 python bench.py --no-cpu-baseline --steps 10 --warmup 3 "$@" > gpurun_out/r02d_$tag.json 2> gpurun_out/r02d_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02d_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'])" || tail -3 gpurun_out/r02d_$tag.err; }
run chr14_flat cur
DBG_SCATTER_TWO_LEVEL=0 run chr14_one cur
run chr14_bucket bucket
run chr14_fp11 cur --fine-p 11
run bbee_blk cur --config bumblebee
run bbee_gen gen63 --config bumblebee
DBG_SCATTER_TWO_LEVEL=0 run bbee_one cur --config bumblebee

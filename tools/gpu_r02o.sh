#!/bin/bash
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
timeout 900 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02o_pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/r02o_pytest.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$V/$lib/libdbg.so timeout 900 python bench.py --no-cpu-baseline --steps 10 --warmup 3 "$@" > gpurun_out/r02o_$tag.json 2> gpurun_out/r02o_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02o_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], round(d['roofline']['frac'],3), d['roofline']['onchip']['stale'], d['roofline']['traffic'])" 2>/dev/null || tail -3 gpurun_out/r02o_$tag.err; }
run chr14_cur cur
run chr14_old old
run bbee_cur cur --config bumblebee --steps 5
run bbee_old old --config bumblebee --steps 5
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:'^scatter_kernel' -s 3 -c 1 -o gpurun_out/r02o_chr14_scatter1 -f \
    python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r02o_ncu.log 2>&1; echo "ncu=$?"
timeout 600 python bench.py --impl reference --steps 5 --warmup 2 > gpurun_out/r02o_reference.json 2> gpurun_out/r02o_reference.err; echo ref=$?; head -c 300 gpurun_out/r02o_reference.json

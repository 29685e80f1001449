#!/bin/bash
# r02r: parity of the warp MSP + 16-byte-load probe; K = 63 step-2 A/B; ncu source capture of msp_warp_kernel
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
timeout 900 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02r_pytest.log 2>&1; echo pytest=$?; tail -3 gpurun_out/r02r_pytest.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$lib timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02r_$tag.json 2> gpurun_out/r02r_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02r_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], d['stats']['checksum'])" 2>/dev/null || tail -3 gpurun_out/r02r_$tag.err; }
run bbee_cur paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 5 --config bumblebee
run bbee_h0 $V/h0/libdbg.so --steps 5 --config bumblebee
timeout 900 ncu --set full --import-source on --clock-control none -k regex:'msp_warp_kernel' -s 1 -c 1 -o gpurun_out/r02r_chr14_mspwarp -f \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/r02r_ncu.log 2>&1; echo "ncu=$?"

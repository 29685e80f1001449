#!/bin/bash
# r02z2: two-level scatter tile size A/B (records per thread 6/3 default vs 8/4 and 4/2); ncu of both levels
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$lib timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02z2_$tag.json 2> gpurun_out/r02z2_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02z2_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], d['stats']['checksum'])" 2>/dev/null || tail -3 gpurun_out/r02z2_$tag.err; }
run chr14_t6 paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 10
run chr14_t8 $V/t8/libdbg.so --steps 10
run chr14_t4 $V/t4/libdbg.so --steps 10
run bbee_t6 paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 5 --config bumblebee
run bbee_t8 $V/t8/libdbg.so --steps 5 --config bumblebee
timeout 900 ncu --set full --import-source on --clock-control none -k regex:'ts_level' -s 2 -c 2 -o gpurun_out/r02z2_ts -f \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/r02z2_ncu.log 2>&1; echo "ncu=$?"

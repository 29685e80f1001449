#!/bin/bash
# r02t: on-chip kernel A/B -- dynamic warp-window claiming (DBG_DYN_WIN) vs static windows
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$lib timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02t_$tag.json 2> gpurun_out/r02t_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02t_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], d['stats']['checksum'])" 2>/dev/null || tail -3 gpurun_out/r02t_$tag.err; }
run bbee_base paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 5 --config bumblebee
run bbee_dyn $V/dyn/libdbg.so --steps 5 --config bumblebee
run chr14_base paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 10
run chr14_dyn $V/dyn/libdbg.so --steps 10
run bbee_base2 paper_conf_icdcs_qiul17_b200/lib/libdbg.so --steps 5 --config bumblebee
run bbee_dyn2 $V/dyn/libdbg.so --steps 5 --config bumblebee

#!/bin/bash
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/r02l_smoke.log 2>&1; echo smoke=$?; tail -1 gpurun_out/r02l_smoke.log
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$V/$lib/libdbg.so timeout 900 python bench.py --no-cpu-baseline --steps 10 --warmup 3 "$@" > gpurun_out/r02l_$tag.json 2> gpurun_out/r02l_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02l_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], round(d['roofline']['frac'],3))" 2>/dev/null || tail -3 gpurun_out/r02l_$tag.err; }
for v in base m6 m6d32 m7d28; do run chr14_$v $v; done
run bbee base --config bumblebee --steps 5

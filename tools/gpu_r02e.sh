#!/bin/bash
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
timeout 600 python -m pytest tests/test_gpu_multi.py tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/r02e_pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/r02e_pytest.log
timeout 600 python tools/scatter_probe.py 295e6 1579008 > gpurun_out/r02e_probe_chr14.txt 2>&1; cat gpurun_out/r02e_probe_chr14.txt
timeout 600 python tools/scatter_probe.py 21.8e6 116736 > gpurun_out/r02e_probe_ecoli.txt 2>&1; cat gpurun_out/r02e_probe_ecoli.txt
run() { tag=$1; lib=$2; shift 2; DBG_SCATTER_TWO_LEVEL=0 DBG_LIB_PATH=$V/$lib/libdbg.so timeout 900 python bench.py --no-cpu-baseline --steps 5 --warmup 3 "$@" > gpurun_out/r02e_$tag.json 2> gpurun_out/r02e_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02e_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'])" 2>/dev/null || tail -3 gpurun_out/r02e_$tag.err; }
run bbee_blk cur --config bumblebee
run bbee_gen gen63 --config bumblebee

#!/bin/bash
# r02u: on-chip kernel A/B -- balanced extraction (DBG_XBAL) with/without dynamic windows; parity of both
mkdir -p gpurun_out
V=paper_conf_icdcs_qiul17_b200/lib/variants
for v in xbal; do
  DBG_LIB_PATH=$V/$v/libdbg.so timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/r02u_pytest_$v.log 2>&1; echo "pytest $v=$?"; tail -1 gpurun_out/r02u_pytest_$v.log
done
run() { tag=$1; lib=$2; shift 2; DBG_LIB_PATH=$lib timeout 900 python bench.py --no-cpu-baseline --warmup 3 "$@" > gpurun_out/r02u_$tag.json 2> gpurun_out/r02u_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02u_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], d['stats']['checksum'])" 2>/dev/null || tail -3 gpurun_out/r02u_$tag.err; }
for c in "bbee --config bumblebee --steps 5" "chr14 --steps 10"; do
  set -- $c; n=$1; shift
  run ${n}_base paper_conf_icdcs_qiul17_b200/lib/libdbg.so "$@"
  run ${n}_xbal $V/xbal/libdbg.so "$@"
  run ${n}_base2 paper_conf_icdcs_qiul17_b200/lib/libdbg.so "$@"
  run ${n}_xbal2 $V/xbal/libdbg.so "$@"
done

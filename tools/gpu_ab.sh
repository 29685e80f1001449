# same-box A/B of kernel variants (tools/build_variants.py) and runtime switches
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "two_level or tiny or smem or low_count or overflow or auto_refine or full_size" > gpurun_out/ab_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/ab_tests.log
run() {  # name, env...
  local name=$1; shift
  env "$@" timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 > gpurun_out/ab_$name.json
  python -c "
import json; d=json.load(open('gpurun_out/ab_$name.json'))
print('$name', round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'])"
}
V=paper_conf_icdcs_qiul17_b200/lib/variants
for rep in 1 2; do
run v0w DBG_LIB_PATH=$V/v0/libdbg.so DBG_GROUPS_WINDOW=1 DBG_SCATTER_ONE_LEVEL=1
run v1w DBG_LIB_PATH=$V/v1/libdbg.so DBG_GROUPS_WINDOW=1 DBG_SCATTER_ONE_LEVEL=1
run v2w DBG_LIB_PATH=$V/v2/libdbg.so DBG_GROUPS_WINDOW=1 DBG_SCATTER_ONE_LEVEL=1
run v3w DBG_LIB_PATH=$V/v3/libdbg.so DBG_GROUPS_WINDOW=1 DBG_SCATTER_ONE_LEVEL=1
run v1g DBG_LIB_PATH=$V/v1/libdbg.so DBG_SCATTER_ONE_LEVEL=1
run v0g DBG_LIB_PATH=$V/v0/libdbg.so DBG_SCATTER_ONE_LEVEL=1
run v1g2 DBG_LIB_PATH=$V/v1/libdbg.so
done

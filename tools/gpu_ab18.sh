# same-box A/B: scatter variants (sc0 default minB 6; sc1 minB 4; sc2 minB 4 + cursors at the record offsets)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
run() {  # name, env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --steps 6 --warmup 3 --no-cpu-baseline "${ARGS[@]}" 2>/dev/null | tail -1 > gpurun_out/ab18_$name.json
  python -c "
import json; d=json.load(open('gpurun_out/ab18_$name.json'))
print('$name', d['config']['workload'], round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['breakdown_ms'].items()}, round(d['roofline']['frac'],3), d['invariants_ok'])"
}
V=paper_conf_icdcs_qiul17_b200/lib/variants
ARGS=()
for rep in 1 2; do for m in sc0 sc1 sc2; do run $m DBG_LIB_PATH=$V/$m/libdbg.so; done; done
DBG_LIB_PATH=$V/sc2/libdbg.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stream.py -m gpu -x -q 2>&1 | tail -1
ARGS=(--config chr14 --steps 4)
for m in sc0 sc2; do run ${m}_chr14 DBG_LIB_PATH=$V/$m/libdbg.so; done

# same-box A/B: evict-first stores: scatter (st1), MSP staging (st2), both (st3) vs st0
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
run() {  # name, env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --steps 6 --warmup 3 --no-cpu-baseline "${ARGS[@]}" 2>/dev/null | tail -1 > gpurun_out/ab19_$name.json
  python -c "
import json; d=json.load(open('gpurun_out/ab19_$name.json'))
print('$name', d['config']['workload'], round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['breakdown_ms'].items()}, round(d['roofline']['frac'],3), d['invariants_ok'])"
}
V=paper_conf_icdcs_qiul17_b200/lib/variants
ARGS=()
for rep in 1 2; do for m in st0 st1 st2 st3; do run $m DBG_LIB_PATH=$V/$m/libdbg.so; done; done
DBG_LIB_PATH=$V/st3/libdbg.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "tiny or ragged or msp or register or two_level" 2>&1 | tail -1
ARGS=(--config chr14 --steps 4)
for m in st0 st3; do run ${m}_chr14 DBG_LIB_PATH=$V/$m/libdbg.so; done

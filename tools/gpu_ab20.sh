# same-box A/B: on-chip kernel with compile-time K (kc1) vs runtime K (kc0)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
run() {  # name, env...
  local name=$1; shift
  env "$@" timeout 900 python bench.py --no-cpu-baseline "${ARGS[@]}" 2>/dev/null | tail -1 > gpurun_out/ab20_$name.json
  python -c "
import json; d=json.load(open('gpurun_out/ab20_$name.json'))
print('$name', d['config']['workload'], round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['breakdown_ms'].items()}, round(d['roofline']['frac'],3), d['invariants_ok'])"
}
V=paper_conf_icdcs_qiul17_b200/lib/variants
ARGS=(--steps 6 --warmup 3)
for rep in 1 2; do for m in kc0 kc1; do run $m DBG_LIB_PATH=$V/$m/libdbg.so; done; done
DBG_LIB_PATH=$V/kc1/libdbg.so timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "tiny or ragged or smem or split or hot or full_size or low_count or fine" 2>&1 | tail -1
ARGS=(--config bumblebee --steps 3 --warmup 3)
for m in kc0 kc1; do run ${m}_bbee DBG_LIB_PATH=$V/$m/libdbg.so; done

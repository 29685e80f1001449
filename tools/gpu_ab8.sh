# same-box A/B: MSP flush with compile-time K (mk) vs HEAD (base); chr14 refine
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
run() {  # name, env...
  local name=$1; shift
  env "$@" timeout 400 python bench.py --steps 6 --warmup 3 --no-cpu-baseline "${ARGS[@]}" 2>/dev/null | tail -1 > gpurun_out/ab8_$name.json
  python -c "
import json; d=json.load(open('gpurun_out/ab8_$name.json'))
print('$name', d['config']['workload'], round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['config']['refine'], d['config']['kmer_placement'], d['invariants_ok'])"
}
V=paper_conf_icdcs_qiul17_b200/lib/variants
ARGS=()
for rep in 1 2; do for m in base mk; do run $m DBG_LIB_PATH=$V/$m/libdbg.so; done; done
DBG_LIB_PATH=$V/mk/libdbg.so timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "register_blocked or msp or tiny or ragged or long or edge or overlapped or two_level" 2>&1 | tail -1
ARGS=(--config chr14 --steps 4)
run chr14_auto DBG_LIB_PATH=$V/mk/libdbg.so
ARGS=(--config chr14 --steps 4 --refine 1700)
run chr14_r1700 DBG_LIB_PATH=$V/mk/libdbg.so
ARGS=(--config chr14 --steps 4 --refine 2400)
run chr14_r2400 DBG_LIB_PATH=$V/mk/libdbg.so
ARGS=(--config chr14 --steps 4 --fine-p 12)
run chr14_fp12 DBG_LIB_PATH=$V/mk/libdbg.so

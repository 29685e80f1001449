# same-box A/B of msp_block_kernel variants
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
run() {  # name, env...
  local name=$1; shift
  env "$@" timeout 300 python bench.py --steps 8 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 > gpurun_out/ab2_$name.json
  python -c "
import json; d=json.load(open('gpurun_out/ab2_$name.json'))
print('$name', round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'])"
}
V=paper_conf_icdcs_qiul17_b200/lib/variants
for rep in 1 2; do
for m in m0 m1 m2 m3 m4; do run $m DBG_LIB_PATH=$V/$m/libdbg.so; done
done
for m in m0 m1 m3; do DBG_LIB_PATH=$V/$m/libdbg.so timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "register_blocked or msp or tiny" 2>&1 | tail -1; done

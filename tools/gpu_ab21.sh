# same-box A/B: generic MSP kernel with 64-bit P-mer codes flushing every 16 bases with 18 descriptors
# (m1, 3 CTAs/SM) vs every 32 bases with 40 (m0); bumblebee (K = 63, P = 19) full size + GPU parity on m1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
run() {  # name, env...
  local name=$1; shift
  env "$@" timeout 900 python bench.py --no-cpu-baseline "${ARGS[@]}" 2>/dev/null | tail -1 > gpurun_out/ab21_$name.json
  python -c "
import json; d=json.load(open('gpurun_out/ab21_$name.json'))
print('$name', d['config']['workload'], round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['breakdown_ms'].items()}, round(d['roofline']['frac'],3), d['invariants_ok'])"
}
V=paper_conf_icdcs_qiul17_b200/lib/variants
DBG_LIB_PATH=$V/m1/libdbg.so timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -1
ARGS=(--config bumblebee --steps 3 --warmup 3)
for rep in 1 2; do for m in m0 m1; do run ${m}_bbee DBG_LIB_PATH=$V/$m/libdbg.so; done; done

# same-box A/B: pass-1 ranks (DBG_MSP_RANK=1: returning record-counter atomics in MSP, atomic-free scatter) vs rank atomics in the scatter
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
run() {  # name, env...
  local name=$1; shift
  env "$@" timeout 600 python bench.py --steps 6 --warmup 3 --no-cpu-baseline "${ARGS[@]}" 2>/dev/null | tail -1 > gpurun_out/ab17_$name.json
  python -c "
import json; d=json.load(open('gpurun_out/ab17_$name.json'))
print('$name', d['config']['workload'], round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['breakdown_ms'].items()}, round(d['roofline']['frac'],3), round(d['e2e']['value']/1e9,3), d['invariants_ok'])"
}
DBG_MSP_RANK=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_stream.py -m gpu -x -q 2>&1 | tail -2
ARGS=()
for rep in 1 2; do run rk0 DBG_MSP_RANK=0; run rk1 DBG_MSP_RANK=1; done
ARGS=(--config chr14 --steps 4)
run rk0_chr14 DBG_MSP_RANK=0; run rk1_chr14 DBG_MSP_RANK=1

# same-box A/B: previous commit vs the working tree (MSP one-reload-per-block + one flush site, scatter defaults)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
run() {  # name, env...
  local name=$1; shift
  env "$@" timeout 300 python bench.py --steps 8 --warmup 3 --no-cpu-baseline 2>/dev/null | tail -1 > gpurun_out/ab5_$name.json
  python -c "
import json; d=json.load(open('gpurun_out/ab5_$name.json'))
print('$name', round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['config']['smem_slots'], d['invariants_ok'])"
}
V=paper_conf_icdcs_qiul17_b200/lib/variants
for rep in 1 2; do for m in prev cur; do run $m DBG_LIB_PATH=$V/$m/libdbg.so; done; done
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "register_blocked or msp or tiny or ragged or long or edge or overlapped" 2>&1 | tail -1

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
# round-1 closing measurements (r01h): tests, smoke, bench lines (ecoli with cpu_baseline, chr14, bumblebee),
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/h_smoke.log 2>&1; echo smoke=$?
# reference arm, launch list, ncu full captures of the three step kernels
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/h_tests.log 2>&1; echo "tests=$?"; tail -2 gpurun_out/h_tests.log
timeout 300 python bench.py --steps 10 --warmup 3 > gpurun_out/h_bench_ecoli.json 2> gpurun_out/h_bench_ecoli.err; echo bench=$?
timeout 900 python bench.py --config chr14 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/h_bench_chr14.json 2> gpurun_out/h_bench_chr14.err; echo chr14=$?
timeout 1200 python bench.py --config bumblebee --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/h_bench_bbee.json 2> gpurun_out/h_bench_bbee.err; echo bbee=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/h_reference.json 2> gpurun_out/h_reference.err; echo ref=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/h_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches=$?
for k in smem_subgraph msp_block scatter_kernel; do
timeout 900 ncu --set full --import-source on --clock-control none -k regex:$k -s 3 -c 1 -o gpurun_out/h_$k -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/h_ncu_$k.log 2>&1; echo "ncu $k=$?"
done

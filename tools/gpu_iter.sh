# one build -> measure iteration: GPU parity suite, ecoli bench, ncu full capture of the on-chip kernel
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/it_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/it_tests.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/it_bench.json 2> gpurun_out/it_bench.err; echo "bench rc=$?"
python - <<'PY'
import json
d=json.loads(open('gpurun_out/it_bench.json').read().strip().splitlines()[-1])
print(round(d['value']/1e9,3),'G/s step', round(d['ms_per_step'],3),'ms; kernel', round(d['roofline']['kernel_ms'],3),'ms frac',round(d['roofline']['frac'],3), d['breakdown_ms'], 'inv', d['invariants_ok'])
PY
if [ "${NCU:-1}" = 1 ]; then
timeout 600 ncu --set full --import-source on --clock-control none -k regex:smem_subgraph -s 3 -c 1 -o gpurun_out/it_smem -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/it_ncu.log 2>&1; echo "ncu rc=$?"
fi

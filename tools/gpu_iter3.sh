# build -> targeted GPU parity -> full GPU suite -> ecoli + chr14 bench lines
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "two_level or register_blocked or tiny or ragged or smem" > gpurun_out/it_tests_a.log 2>&1; echo "tests_a rc=$?"; tail -3 gpurun_out/it_tests_a.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/it_bench.json 2> gpurun_out/it_bench.err; echo "bench rc=$?"
timeout 900 python bench.py --config chr14 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/it_chr14.json 2> gpurun_out/it_chr14.err; echo "chr14 rc=$?"
python - <<'PY'
import json
for f in ['gpurun_out/it_bench.json','gpurun_out/it_chr14.json']:
    try:
        d=json.loads(open(f).read().strip().splitlines()[-1])
        print(f, round(d['value']/1e9,3),'G/s step', round(d['ms_per_step'],3),'ms; kernel', round(d['roofline']['kernel_ms'],3),'ms frac',round(d['roofline']['frac'],3), d['breakdown_ms'], 'inv', d['invariants_ok'], 'e2e', round(d['e2e']['value']/1e9,3))
    except Exception as e: print(f, 'ERR', e)
PY
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/it_tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/it_tests.log

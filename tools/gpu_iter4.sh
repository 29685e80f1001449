# build -> targeted GPU parity -> ecoli + chr14 bench -> ncu of msp/scatter/smem
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "two_level or register_blocked or tiny or ragged or smem or low_count or overflow or full_size" > gpurun_out/it_tests_a.log 2>&1; echo "tests_a rc=$?"; tail -3 gpurun_out/it_tests_a.log
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
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/it_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo "launches rc=$?"
for k in msp_block smem_subgraph; do
timeout 900 ncu --set full --import-source on --clock-control none -k regex:$k -s 3 -c 1 -o gpurun_out/p4_$k -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/p4_$k.log 2>&1; echo "$k rc=$?"
done

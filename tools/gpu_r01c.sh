# round-1 closing measurements: tests, bench (with cpu_baseline), launch list, ncu full captures,
# larger configs, reference arm, f1 sweep
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/c_smoke.log 2>&1; echo smoke=$?
timeout 300 python bench.py --steps 10 --warmup 3 > gpurun_out/c_bench_ecoli.json 2> gpurun_out/c_bench_ecoli.err; echo bench=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/c_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:smem_subgraph -s 3 -c 1 -o gpurun_out/c_smem -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu1=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:msp_kernel -s 3 -c 1 -o gpurun_out/c_msp -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu2=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:scatter_kernel -s 3 -c 1 -o gpurun_out/c_scatter -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo ncu3=$?
timeout 900 python bench.py --config chr14 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/c_bench_chr14.json 2>&1; echo chr14=$?
timeout 1200 python bench.py --config bumblebee --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/c_bench_bbee.json 2>&1; echo bbee=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/c_reference.json 2>&1; echo ref=$?
bash tools/f1_sweep.sh > gpurun_out/c_f1_sweep.jsonl; echo sweep=$?

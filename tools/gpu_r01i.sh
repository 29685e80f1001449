python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
# round-1 closing measurements (r01i): tests, smoke, bench lines (ecoli with cpu_baseline, chr14, bumblebee),
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/i_smoke.log 2>&1; echo smoke=$?
# reference arm, launch list, ncu full captures of the three step kernels
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/i_tests.log 2>&1; echo "tests=$?"; tail -2 gpurun_out/i_tests.log
timeout 300 python bench.py --steps 10 --warmup 3 > gpurun_out/i_bench_ecoli.json 2> gpurun_out/i_bench_ecoli.err; echo bench=$?
timeout 900 python bench.py --config chr14 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/i_bench_chr14.json 2> gpurun_out/i_bench_chr14.err; echo chr14=$?
timeout 1200 python bench.py --config bumblebee --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/i_bench_bbee.json 2> gpurun_out/i_bench_bbee.err; echo bbee=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/i_reference.json 2> gpurun_out/i_reference.err; echo ref=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/i_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches=$?
for k in smem_subgraph msp_block scatter_kernel; do
timeout 900 ncu --set full --import-source on --clock-control none -k regex:$k -s 3 -c 1 -o gpurun_out/i_$k -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/i_ncu_$k.log 2>&1; echo "ncu $k=$?"
done

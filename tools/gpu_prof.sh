# launch list + full ncu capture of the two top kernels, then the larger configs
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/launches_bench.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:smem_subgraph -s 3 -c 1 -o gpurun_out/prof_smem python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_smem.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:msp_kernel -s 3 -c 1 -o gpurun_out/prof_msp python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_msp.log 2>&1
timeout 900 python bench.py --config chr14 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/chr14.json 2> gpurun_out/chr14.err
timeout 1200 python bench.py --config bumblebee --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bbee.json 2> gpurun_out/bbee.err
ls -la gpurun_out

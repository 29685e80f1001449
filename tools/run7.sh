python -m pytest tests -m gpu -x -q --timeout 900 > gpurun_out/t7.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t7.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ecoli7.json 2> gpurun_out/ecoli7.err
timeout 600 python bench.py --config chr14 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/chr14_7.json 2> gpurun_out/chr14_7.err
timeout 900 ncu --set full --import-source on --clock-control none -k regex:smem_subgraph -s 2 -c 1 -o gpurun_out/prof_smem7 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu7.log 2>&1

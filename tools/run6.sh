python -m pytest tests -m gpu -x -q --timeout 900 > gpurun_out/t6.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t6.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --fine-p 12 > gpurun_out/ecoli6_fp12.json 2> gpurun_out/ecoli6_fp12.err
timeout 600 python bench.py --config chr14 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/chr14_6.json 2> gpurun_out/chr14_6.err
timeout 900 ncu --set full --import-source on --clock-control none -k regex:smem_subgraph -s 2 -c 1 -o gpurun_out/prof_smem6 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu6.log 2>&1

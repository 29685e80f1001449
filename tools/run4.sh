python -m pytest tests -m gpu -x -q --timeout 900 > gpurun_out/t4.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t4.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ecoli4.json 2> gpurun_out/ecoli4.err
for FP in 12 13; do timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --fine-p $FP > gpurun_out/ecoli4_fp$FP.json 2> gpurun_out/ecoli4_fp$FP.err; done
for FP in 13 14 15; do timeout 600 python bench.py --config chr14 --fine-p $FP --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/chr14_4_fp$FP.json 2> gpurun_out/chr14_4_fp$FP.err; done

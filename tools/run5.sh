python -m pytest tests -m gpu -x -q --timeout 900 -k "fine or tiny or ragged" > gpurun_out/t5.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t5.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --fine-p 12 > gpurun_out/ecoli5_fp12.json 2> gpurun_out/ecoli5_fp12.err
for FP in 13 15; do timeout 600 python bench.py --config chr14 --fine-p $FP --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/chr14_5_fp$FP.json 2> gpurun_out/chr14_5_fp$FP.err; done

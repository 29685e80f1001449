python -m pytest tests -m gpu -x -q --timeout 900 > gpurun_out/t3.log 2>&1; echo "pytest rc=$?" >> gpurun_out/t3.log
for P in 11 13 15 17 19 21; do
  timeout 600 python bench.py --config chr14 --p $P --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/chr14_p$P.json 2> gpurun_out/chr14_p$P.err
done

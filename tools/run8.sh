for C in 0 1 2 4; do DBG_SMEM_CTAS=$C timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/ecoli8_c$C.json 2> gpurun_out/ecoli8_c$C.err; done
for C in 2 4; do DBG_SMEM_CTAS=$C timeout 600 python bench.py --config chr14 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/chr14_8_c$C.json 2> gpurun_out/chr14_8_c$C.err; done

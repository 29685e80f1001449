# on-chip kernel variants: CTAs per SM (DBG_SMEM_CTAS) and load ratio alpha
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for c in 0 1 2 4; do
  DBG_SMEM_CTAS=$c timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/var_ctas$c.json 2>&1
done
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --alpha 0.8 > gpurun_out/var_alpha08.json 2>&1
timeout 600 python -m pytest tests -m gpu -x -q -k "low_count" > gpurun_out/t_filter.log 2>&1

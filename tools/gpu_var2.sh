# on-chip kernel variants (DBG_SMEM_CTAS) after a build; parity of the variant on the smem tests
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for c in 0 3 1; do
  DBG_SMEM_CTAS=$c timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/var_ctas$c.json 2>&1
  python - $c <<'PY'
import json,sys
d=json.loads(open(f'gpurun_out/var_ctas{sys.argv[1]}.json').read().strip().splitlines()[-1])
print('ctas',sys.argv[1], round(d['value']/1e9,3),'G/s step', round(d['ms_per_step'],3),'ms; kernel', round(d['roofline']['kernel_ms'],3),'frac',round(d['roofline']['frac'],3), d['breakdown_ms'], d['config']['smem_slots'], d['config']['refine'], d['config']['kmer_placement'])
PY
done
DBG_SMEM_CTAS=3 timeout 600 python -m pytest tests -m gpu -x -q -k "smem or tiny or ragged or split or fine" > gpurun_out/t_var.log 2>&1; tail -2 gpurun_out/t_var.log

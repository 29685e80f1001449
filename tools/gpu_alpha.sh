# alpha sweep (paper: lambda = 2, alpha in [0.5, 0.8]) on the E. coli config
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for a in 0.5 0.65 0.8; do
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --alpha $a 2>/dev/null | tail -1 > gpurun_out/alpha_$a.json
python -c "
import json; d=json.load(open('gpurun_out/alpha_$a.json'))
print('alpha $a', round(d['value']/1e9,3), 'G/s', round(d['ms_per_step'],3), 'ms', d['breakdown_ms'], 'frac', round(d['roofline']['frac'],3), d['config']['refine'], d['config']['kmer_placement'])"
done

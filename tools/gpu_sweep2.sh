# build -> MSP/on-chip parity -> refine x fine_p sweep on E. coli (greedy group packing)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -k "register_blocked or msp or tiny or ragged or two_level or overlapped" > gpurun_out/sw_tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/sw_tests.log
run() {  # name, args...
  local name=$1; shift
  timeout 300 python bench.py --steps 8 --warmup 3 --no-cpu-baseline "$@" 2>/dev/null | tail -1 > gpurun_out/sw_$name.json
  python -c "
import json; d=json.load(open('gpurun_out/sw_$name.json'))
c=d['config']; print('$name', round(d['ms_per_step'],3), 'ms', {k: round(v,3) for k,v in d['breakdown_ms'].items()}, 'refine', c['refine'], 'fine_p', c['fine_p'], c['kmer_placement'], d['invariants_ok'])"
}
run auto
for fp in 11 12 13; do for rf in 70 140 280; do run f${fp}_r$rf --fine-p $fp --refine $rf; done; done
run auto2

#!/bin/bash
mkdir -p gpurun_out
run() { tag=$1; shift; timeout 900 python bench.py --no-cpu-baseline --steps 5 --warmup 3 "$@" > gpurun_out/r02i_$tag.json 2> gpurun_out/r02i_$tag.err
  python -c "import json,sys; d=json.load(open('gpurun_out/r02i_$tag.json')); print('$tag', round(d['value']/1e9,3), round(d['ms_per_step'],3), {k: round(v,3) for k,v in d['breakdown_ms'].items()}, d['invariants_ok'], round(d['roofline']['frac'],3), d['config']['fine_partitions'], d['config']['kmer_placement'])" 2>/dev/null || tail -3 gpurun_out/r02i_$tag.err; }
run chr14_a08 --alpha 0.8
run chr14_a065 --alpha 0.65
run ecoli_a08 --config ecoli --alpha 0.8
run bbee_a08 --config bumblebee --alpha 0.8
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:msp_kernel -s 3 -c 1 -o gpurun_out/r02i_bbee_msp -f \
    python bench.py --config bumblebee --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r02i_ncu.log 2>&1; echo "ncu=$?"

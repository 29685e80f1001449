#!/bin/bash
# Row f1: P / NP sweep on the E. coli-shaped config (Fig. 6-7 / Table II analogue).
# usage: tools/f1_sweep.sh > gpurun_out/f1_sweep.jsonl
for p in 9 11 13 15; do for np in 16 128 512 2048; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --p $p --np $np 2>/dev/null | tail -1
done; done

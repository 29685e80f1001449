#!/bin/bash
# r02z7: the final state -- full-size parity (whole E. coli graph; chr14, bumblebee sampled partitions) and an
# ncu capture of the 4-CTA warp MSP kernel on bumblebee
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_fullsize.py -x -q > gpurun_out/r02z7_fullsize.log 2>&1; echo fullsize=$?; tail -1 gpurun_out/r02z7_fullsize.log
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:msp_warp -s 3 -c 1 -o gpurun_out/r02z7_bbee_msp_warp -f \
    python bench.py --config bumblebee --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/r02z7_ncu.log 2>&1; echo "ncu=$?"

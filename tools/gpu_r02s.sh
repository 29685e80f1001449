#!/bin/bash
# r02s: parity after the MSP dispatch change; ncu source-level captures of the on-chip kernel
# (chr14 K = 31, bumblebee K = 63) and of msp_warp_kernel (K = 63)
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_fullsize.py > gpurun_out/r02s_pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/r02s_pytest.log
timeout 900 ncu --set full --import-source on --clock-control none -k regex:'smem_subgraph_kernel' -c 1 -o gpurun_out/r02s_chr14_smem -f \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/r02s_ncu1.log 2>&1; echo "ncu1=$?"
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:'smem_subgraph_kernel|msp_warp_kernel' -c 2 -o gpurun_out/r02s_bbee -f \
    python bench.py --steps 1 --warmup 1 --no-cpu-baseline --config bumblebee > gpurun_out/r02s_ncu2.log 2>&1; echo "ncu2=$?"

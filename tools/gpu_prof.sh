#!/bin/bash
# Profiles one bench workload on the GPU box: the launch list (gpu__time_duration, cold-cache
# serialised) and one `ncu --set full` capture per named kernel (the launch of the first timed step).
#   tools/gpu_prof.sh TAG CONFIG "kernel_regex1 kernel_regex2 ..." [extra bench args]
TAG=$1; CFG=$2; KERNELS=$3; shift 3
mkdir -p gpurun_out
python -m paper_conf_icdcs_qiul17_b200.build > gpurun_out/${TAG}_build.log 2>&1 || { cat gpurun_out/${TAG}_build.log; exit 1; }
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${TAG}_launches.csv \
  python bench.py --config $CFG --steps 2 --warmup 3 --no-cpu-baseline "$@" > /dev/null 2>&1; echo launches=$?
for k in $KERNELS; do
  timeout 1200 ncu --set full --import-source on --clock-control none -k regex:$k -s 3 -c 1 -o gpurun_out/${TAG}_$k -f \
    python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline "$@" > gpurun_out/${TAG}_ncu_$k.log 2>&1; echo "ncu $k=$?"
done

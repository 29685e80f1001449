# K = 63 evidence for round 2: ncu full captures of the on-chip kernel and the generic MSP kernel on
# bumblebee (scale 0.25: same per-partition shapes, fewer reads), launch list of the same run
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { cat gpurun_out/build.log; exit 1; }
for k in smem_subgraph msp_kernel; do
timeout 900 ncu --set full --import-source on --clock-control none -k regex:$k -s 1 -c 1 -o gpurun_out/j_bbee_$k -f python bench.py --config bumblebee --scale 0.25 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/j_ncu_$k.log 2>&1; echo "ncu $k=$?"
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/j_bbee_launches.csv python bench.py --config bumblebee --scale 0.25 --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches=$?

#!/bin/bash
# Round-closing measurements: build + smoke, every GPU test, bench lines (chr14 with cpu_baseline,
# bumblebee, E. coli, the reference arm), the chr14 launch list, ncu full captures of the step's
# kernels (chr14, bumblebee), compute-sanitizer over every tier.   tools/gpu_final.sh TAG
T=${1:-r02z}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/${T}_smoke.log 2>&1; echo smoke=$?; tail -1 gpurun_out/${T}_smoke.log
timeout 2400 python -m pytest tests -m gpu -q --durations=15 > gpurun_out/${T}_pytest.log 2>&1; echo pytest=$?; tail -3 gpurun_out/${T}_pytest.log
timeout 900 python bench.py > gpurun_out/${T}_bench_chr14.json 2> gpurun_out/${T}_bench_chr14.err; echo chr14=$?
timeout 900 python bench.py --config bumblebee --steps 5 --no-cpu-baseline > gpurun_out/${T}_bench_bbee.json 2> gpurun_out/${T}_bench_bbee.err; echo bbee=$?
timeout 600 python bench.py --config ecoli --no-cpu-baseline > gpurun_out/${T}_bench_ecoli.json 2> gpurun_out/${T}_bench_ecoli.err; echo ecoli=$?
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/${T}_reference.json 2> gpurun_out/${T}_reference.err; echo ref=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/${T}_launches.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches=$?
for k in smem_subgraph msp_block ts_level_a ts_level_b; do
  timeout 1200 ncu --set full --import-source on --clock-control none -k regex:$k -s 3 -c 1 -o gpurun_out/${T}_chr14_$k -f \
    python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/${T}_ncu_chr14_$k.log 2>&1; echo "ncu chr14 $k=$?"
done
for k in smem_subgraph msp_warp; do
  timeout 1500 ncu --set full --import-source on --clock-control none -k regex:$k -s 3 -c 1 -o gpurun_out/${T}_bbee_$k -f \
    python bench.py --config bumblebee --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/${T}_ncu_bbee_$k.log 2>&1; echo "ncu bbee $k=$?"
done
timeout 1200 python tools/human_run.py > gpurun_out/${T}_human.json 2> gpurun_out/${T}_human.err; echo human=$?; tail -c 400 gpurun_out/${T}_human.json
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_driver.py > gpurun_out/${T}_san_$tool.log 2>&1
  echo "$tool rc=$?"; tail -1 gpurun_out/${T}_san_$tool.log
done

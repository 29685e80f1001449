#!/bin/bash
# compute-sanitizer over every kernel tier (tools/sanitize_driver.py), one tool per pass.
mkdir -p gpurun_out
python -m paper_conf_icdcs_qiul17_b200.build > /dev/null 2>&1
for tool in memcheck racecheck synccheck initcheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 50 python tools/sanitize_driver.py \
    > gpurun_out/san_$tool.log 2>&1; echo "$tool rc=$?"; tail -4 gpurun_out/san_$tool.log
done

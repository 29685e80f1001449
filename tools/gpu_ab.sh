#!/bin/bash
# Same-box A/B of libdbg.so variants (tools/build_variants.py builds lib/variants/<name>/):
#   tools/gpu_ab.sh TAG CONFIG "variant1 variant2 ..." [extra bench args]
TAG=$1; CFG=$2; VARS=$3; shift 3
mkdir -p gpurun_out
for v in $VARS; do
  DBG_LIB_PATH=paper_conf_icdcs_qiul17_b200/lib/variants/$v/libdbg.so timeout 900 python bench.py --config $CFG \
    --no-cpu-baseline "$@" > gpurun_out/${TAG}_$v.json 2> gpurun_out/${TAG}_$v.err
  python - "$v" gpurun_out/${TAG}_$v.json <<'PY'
import json, sys
try:
    d = json.load(open(sys.argv[2]))
    print(sys.argv[1], round(d["value"] / 1e9, 3), "G/s", round(d["ms_per_step"], 3), "ms",
          {k: round(v, 3) for k, v in d["breakdown_ms"].items()}, "inv", d["invariants_ok"])
except Exception as e:
    print(sys.argv[1], "failed", e)
PY
done

#!/bin/bash
# usage: tools/sweep_smem.sh "<np list>" "<refine list>" [extra]
for np in $1; do for rf in $2; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --np $np --refine $rf --mode smem $3 > gpurun_out/sweeps_${np}_${rf}.log 2>&1
  python - "$np" "$rf" <<'PY'
import json, sys
np_, rf = sys.argv[1], sys.argv[2]
try:
    d = json.loads(open(f"gpurun_out/sweeps_{np_}_{rf}.log").read().strip().splitlines()[-1])
    print(np_, rf, d["config"]["batches"], round(d["value"] / 1e9, 2), "Gk/s", round(d["ms_per_step"], 2), "ms", {k: round(v, 2) for k, v in d["breakdown_ms"].items()}, d["invariants_ok"])
except Exception as e:
    print(np_, rf, "FAIL", open(f"gpurun_out/sweeps_{np_}_{rf}.log").read()[-600:])
PY
done; done

#!/bin/bash
# usage: tools/sweep.sh "<np list>" "<group_slots list>" [extra bench args]
for np in $1; do for gs in $2; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --np $np --group-slots $gs $3 > gpurun_out/sweep_${np}_${gs}.log 2>&1
  python - "$np" "$gs" <<'PY'
import json, sys
np_, gs = sys.argv[1], sys.argv[2]
try:
    d = json.loads(open(f"gpurun_out/sweep_{np_}_{gs}.log").read().strip().splitlines()[-1])
    print(np_, gs, round(d["value"] / 1e9, 2), "Gk/s", round(d["ms_per_step"], 2), "ms", {k: round(v, 2) for k, v in d["breakdown_ms"].items()}, d["invariants_ok"])
except Exception as e:
    print(np_, gs, "FAIL", open(f"gpurun_out/sweep_{np_}_{gs}.log").read()[-400:])
PY
done; done

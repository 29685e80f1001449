#!/bin/bash
# usage: tools/sweep_resident.sh "<np list>" "<budget bytes list>"
for np in $1; do for bud in $2; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --np $np --mode resident --table-budget $bud > gpurun_out/sweepr_${np}_${bud}.log 2>&1
  python - "$np" "$bud" <<'PY'
import json, sys
np_, bud = sys.argv[1], sys.argv[2]
try:
    d = json.loads(open(f"gpurun_out/sweepr_{np_}_{bud}.log").read().strip().splitlines()[-1])
    print(np_, bud, d["config"]["batches"], round(d["value"] / 1e9, 2), "Gk/s", round(d["ms_per_step"], 2), "ms", {k: round(v, 2) for k, v in d["breakdown_ms"].items()}, d["invariants_ok"])
except Exception as e:
    print(np_, bud, "FAIL", open(f"gpurun_out/sweepr_{np_}_{bud}.log").read()[-400:])
PY
done; done

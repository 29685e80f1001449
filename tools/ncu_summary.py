#!/usr/bin/env python
"""Summarise ncu output for profiles/: a launch list (--metrics gpu__time_duration.sum --csv) and
full captures (.ncu-rep, read with `ncu -i ... --page raw --csv` / `--page source --csv`).

    python tools/ncu_summary.py launches gpurun_out/launches.csv > profiles/rNN_launches_summary.json
    python tools/ncu_summary.py full gpurun_out/prof_smem.ncu-rep [...] > profiles/rNN_ncu_full_summary.json
"""
from __future__ import annotations

import collections
import csv
import io
import json
import subprocess
import sys

METRICS = [
    "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sector_hit_rate.pct",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "launch__registers_per_thread", "smsp__inst_executed.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum",
    "sm__cycles_elapsed.avg.per_second", "launch__grid_size", "launch__block_size",
    "launch__shared_mem_per_block_dynamic", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
]


def launches(path: str) -> dict:
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    agg: dict[str, list] = collections.OrderedDict()
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        scale = {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0}.get(r[ui], 1e-6)
        a = agg.setdefault(r[ki][:90], [0, 0.0])
        a[0] += 1
        a[1] += float(r[vi].replace(",", "")) * scale
    tot = sum(a[1] for a in agg.values())
    ks = [{"kernel": n, "launches": c, "total_ms": round(t, 4), "avg_ms": round(t / c, 4), "share": round(t / tot, 4)}
          for n, (c, t) in sorted(agg.items(), key=lambda x: -x[1][1])]
    return {"source": f"ncu --metrics gpu__time_duration.sum --clock-control none ({path}); cold-cache serialised "
                      "launches: compare shares, not absolute times", "total_ms": round(tot, 4), "kernels": ks}


def _ncu_csv(rep: str, *args) -> list[list[str]]:
    out = subprocess.run(["ncu", "-i", rep, *args, "--csv"], capture_output=True, text=True, check=True).stdout
    return list(csv.reader(io.StringIO(out)))


def full(rep: str) -> dict:
    rows = _ncu_csv(rep, "--page", "raw")
    h, units = rows[0], rows[1]
    res = []
    for v in rows[2:]:
        d = {"kernel": v[h.index("Kernel Name")][:90]}
        for m in METRICS:
            if m in h:
                d[m] = f"{v[h.index(m)]} {units[h.index(m)]}".strip()
        st = {n[len("smsp__pcsamp_warps_issue_stalled_"):]: float(v[i] or 0) for i, n in enumerate(h)
              if n.startswith("smsp__pcsamp_warps_issue_stalled_") and not n.endswith("_not_issued")}
        tot = sum(st.values()) or 1.0
        d["stall_share"] = {k: round(x / tot, 3) for k, x in sorted(st.items(), key=lambda x: -x[1])[:8]}
        res.append(d)
    # SASS instruction mix and the hottest stall sites (source page)
    try:
        src = _ncu_csv(rep, "--page", "source", "--print-source", "sass")
        hi = next(i for i, r in enumerate(src) if "Source" in r and "Instructions Executed" in r)
        sh = src[hi]
        si, ni, ie, at = (sh.index("Source"), sh.index("Warp Stall Sampling (All Samples)"),
                          sh.index("Instructions Executed"), sh.index("Avg. Threads Executed"))
        data = [(r[si].strip(), int(r[ni] or 0), int(r[ie] or 0), float(r[at] or 0)) for r in src[hi + 1:]
                if len(r) > ie]
        toti = sum(d[2] for d in data) or 1
        tots = sum(d[1] for d in data) or 1
        mix = collections.Counter()
        for s, _, i, _ in data:
            t = s.split()
            op = (t[1] if t[0].startswith("@") else t[0]).split(".")[0]
            mix[op] += i
        res[0]["sass_mix"] = {o: round(i / toti, 3) for o, i in mix.most_common(12)}
        res[0]["avg_threads_per_warp_inst"] = round(sum(d[2] * d[3] for d in data) / toti, 2)
        res[0]["top_stall_sites"] = [{"sass": s[:70], "stall_share": round(n / tots, 3)}
                                     for s, n, _, _ in sorted(data, key=lambda x: -x[1])[:6]]
    except Exception as e:  # pragma: no cover - report only
        res[0]["source_page_error"] = str(e)
    return {"source": f"ncu --set full --clock-control none --import-source on ({rep})", "kernels": res}


def main():
    mode, paths = sys.argv[1], sys.argv[2:]
    if mode == "launches":
        print(json.dumps(launches(paths[0]), indent=1))
    else:
        out = {"captures": [full(p) for p in paths]}
        print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()

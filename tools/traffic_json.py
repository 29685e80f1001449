#!/usr/bin/env python
"""Writes profiles/traffic.json -- the ncu facts bench.py quotes under roofline.onchip / .traffic --
from `ncu --set full` captures of the on-chip kernel (tools/ncu_summary.py output):

    python tools/traffic_json.py KERNEL_VERSION WORKLOAD KMERS_PER_LAUNCH SUMMARY.json [WORKLOAD ...]
"""
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _num(v: str) -> float:
    """'1.23 Gbyte' / '60.1 %' / '3079 inst' -> base units."""
    m = re.match(r"([-0-9.eE+]+)\s*(\S*)", v.strip())
    x, unit = float(m.group(1)), m.group(2)
    return x * {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "byte": 1.0}.get(unit, 1.0)


def main():
    version = sys.argv[1]
    args = sys.argv[2:]
    path = os.path.join(ROOT, "profiles", "traffic.json")
    out = json.load(open(path)) if os.path.exists(path) else {}
    for i in range(0, len(args), 3):
        name, kmers, summ = args[i], float(args[i + 1]), args[i + 2]
        caps = json.load(open(summ))["captures"]
        k = next(k for c in caps for k in c["kernels"] if "smem_subgraph_kernel" in k["kernel"])
        dram = _num(k["dram__bytes_read.sum"]) + _num(k["dram__bytes_write.sum"])
        wf = _num(k["l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"])
        bc = _num(k["l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"])
        out[name] = {
            "kernel": k["kernel"], "kernel_version": version,
            "dram_bytes_per_launch": dram,
            "dram_bytes_per_kmer": round(dram / kmers, 3),
            "issue_active_pct": round(_num(k["smsp__issue_active.avg.pct_of_peak_sustained_active"]), 2),
            "warps_active_pct": round(_num(k["sm__warps_active.avg.pct_of_peak_sustained_active"]), 2),
            "warp_inst_per_kmer": round(_num(k["smsp__inst_executed.sum"]) / kmers, 3),
            "l2_hit_pct": round(_num(k["lts__t_sector_hit_rate.pct"]), 2),
            "bank_conflict_pct": round(100 * bc / max(wf, 1.0), 2),
            "ncu_ms": round(_num(k["gpu__time_duration.sum"]), 3),
            "stall_share": k.get("stall_share"),
            "source": f"{summ} (ncu --set full --clock-control none, one launch in the bench's launch configuration)",
        }
    json.dump(out, open(path, "w"), indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()

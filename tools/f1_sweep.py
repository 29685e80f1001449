#!/usr/bin/env python
"""Row f1: P / NP sweep on one workload (default chr14) -- the B200 analogues of the paper's Table II
(table size per partition vs NP), Fig. 6 (partition-size skew vs P)
and Fig. 7 (hash time vs NP).  The reads are generated once; each (P, NP) setting
runs the bench's launch configuration (launch_builder: auto refine and fine_p) for a few timed
steps (CUDA events, per-phase events).  One JSON line per setting.

    python tools/f1_sweep.py [--config chr14] [--p 9,11,13,15] [--np 16,32,64,128,256,512,960]
"""
import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_icdcs_qiul17_b200 import encode_reads, launch_builder, _lib  # noqa: E402
from synth import make_config  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="chr14")
    ap.add_argument("--p", default="9,11,13,15")
    ap.add_argument("--np", default="16,32,64,128,256,512,960")
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=2)
    args = ap.parse_args()
    rs = make_config(args.config)
    n_kmers = rs.n_kmers()
    packed = encode_reads(rs.seq, pin=True)
    offsets = torch.from_numpy(rs.offsets.view(np.int64)).pin_memory()
    d_bases, d_off = packed.cuda(), offsets.cuda()
    stream = torch.cuda.current_stream()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for p in [int(x) for x in args.p.split(",")]:
        for np_ in [int(x) for x in args.np.split(",")]:
            b = launch_builder(rs.k, p, np_, n_kmers, device="cuda")
            out_cap = int(0.4 * n_kmers) + (1 << 20)

            def step():
                b.msp(d_bases, d_off, stream)
                b.plan(stream)
                b.reset_output(out_cap, stream)
                b.step2(stream)

            for _ in range(args.warmup):
                step()
            st = _lib.dbg_sync_status(b.d_status, stream)
            b.timer = {}
            ms = []
            for _ in range(args.steps):
                flush.zero_()
                torch.cuda.synchronize()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record(stream)
                step()
                e1.record(stream)
                torch.cuda.synchronize()
                ms.append(e0.elapsed_time(e1))
            phases = {k: round(statistics.mean(a.elapsed_time(c) for a, c in v), 3) for k, v in b.timer.items()}
            b.timer = None
            pk = b.part_kmers
            # K-mers per paper partition (the vertices' pid, reading V): sum of counts per pid
            n = int(b.d_n_out.item())
            rec = b.out[:n * 56].view(torch.int32).view(n, 14)
            paper = torch.bincount(rec[:, 13].long(), weights=rec[:, 4].double(), minlength=np_).cpu().numpy()
            uniq, inv = np.unique(pk, return_inverse=True)
            place = np.array([_lib.dbg_smem_onchip(b.prm, int(n)) for n in uniq])[inv]
            line = {"workload": rs.name, "p": p, "np": np_, "refine": b.refine, "fine_partitions": b.np,
                    "fine_p": b.fine_p or p, "status": st, "ms_per_step": round(statistics.mean(ms), 3),
                    "gkmers_per_s": round(n_kmers / statistics.mean(ms) / 1e6, 2) / 1e3, "phases_ms": phases,
                    "records": int(b.part_records.sum()),
                    "kmers_per_record": round(n_kmers / max(int(b.part_records.sum()), 1), 3),
                    # Table II analogue: the paper's partitions (fine pid mod NP)
                    "paper_part_mean_mkmers": round(float(paper.mean()) / 1e6, 3),
                    "paper_part_max_mkmers": round(float(paper.max()) / 1e6, 3),
                    "paper_table_max_mb": round(_lib.dbg_table_bytes(b.prm, int(paper.max())) / 1e6, 1),
                    "paper_table_max_mb_32B": round(32 * float(paper.max()) / 1e6, 1),
                    # Fig. 6 analogue: skew of the partitions the device works on
                    "paper_max_over_mean": round(float(paper.max() / max(paper.mean(), 1e-9)), 3),
                    "paper_cv": round(float(paper.std() / max(paper.mean(), 1e-9)), 4),
                    "fine_max_over_mean": round(float(pk.max() / max(pk.mean(), 1e-9)), 3),
                    "share_split": round(float(pk[place >= 2].sum()) / n_kmers, 4),
                    "share_global": round(float(pk[place == 0].sum()) / n_kmers, 4)}
            print(json.dumps(line), flush=True)
            del b
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()

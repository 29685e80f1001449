#!/usr/bin/env python
"""Row f2 at the scale it exists for: the whole-human-shaped configuration (BASELINE.json
configs[4]; 3.1 Gbp, 100 bp reads at 30x, K = 31, P = 11, NP = 960), streamed through one GPU by
partition ranges (StreamingBuilder, Sec. III-E), with sampled parity.

    python tools/human_run.py [--scale 0.125] [--budget-gb 12] [--pids 16]

--scale shrinks genome and read count together (same coverage, error rate, read length); 0.125 is
one GPU's share of the 8-GPU run in read count (116 M reads, 8.1 G K-mers).  The graph does not fit
host memory at full scale (12.5 G vertices x 56 B), so the vertices never leave the device in bulk:
a sink keeps, per range, only the records of 16 seeded paper partitions, and the order-independent
checksum, distinct / sum_count / sum_edges are accumulated per range on the device.  Checks:
I1, I2, and the sampled partitions bit-exact against oracle.graph(pids=...) over all reads.
Prints one JSON line.
"""
import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
from paper_conf_icdcs_qiul17_b200 import VERTEX_DTYPE, DbgBuilder, auto_fine_p, auto_refine  # noqa: E402
from paper_conf_icdcs_qiul17_b200.stream import StreamingBuilder, _batches  # noqa: E402
from synth import make_config  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--scale", type=float, default=0.125)
    ap.add_argument("--budget-gb", type=float, default=12.0, help="staging budget per partition range")
    ap.add_argument("--batch-reads", type=int, default=1 << 24)
    ap.add_argument("--pids", type=int, default=16)
    ap.add_argument("--resident", action="store_true", help="keep the packed reads in HBM")
    ap.add_argument("--no-oracle", action="store_true")
    ap.add_argument("--out-frac", type=float, default=0.25, help="output capacity / K-mers of a range")
    args = ap.parse_args()
    t0 = time.time()
    rs = make_config("human", scale=args.scale)
    gen_s = time.time() - t0
    k, p, np_ = rs.k, rs.p, rs.num_partitions
    n_kmers = rs.n_kmers()
    refine = auto_refine(n_kmers, k, p, np_)
    fine_p = auto_fine_p(n_kmers, k, p)
    b = DbgBuilder(k, p, np_, device="cuda", refine=refine, fine_p=fine_p)
    rng = np.random.default_rng(20261017 + np_)
    pids = np.sort(rng.choice(np_, size=args.pids, replace=False))
    d_pids = torch.from_numpy(pids.astype(np.int32)).cuda()
    kept = []

    def sink(d_rec, n):
        rec = d_rec.view(torch.int32).view(n, VERTEX_DTYPE.itemsize // 4)
        m = torch.isin(rec[:, -1], d_pids)
        kept.append(rec[m].contiguous().cpu().numpy().view(VERTEX_DTYPE).reshape(-1))

    t1 = time.time()
    batches = _batches(np.ascontiguousarray(rs.seq), rs.offsets, args.batch_reads)
    enc_s = time.time() - t1
    budget = int(args.budget_gb * (1 << 30) / (4 * b.rec_words))
    sb = StreamingBuilder(b, budget, resident=args.resident)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t2 = time.time()
    e0.record()
    res = sb.run(batches, sort=False, out_frac=args.out_frac, sink=sink)
    e1.record()
    torch.cuda.synchronize()
    wall_s = time.time() - t2
    dev_ms = e0.elapsed_time(e1)
    L = rs.lengths()
    st = res.stats
    out = {"workload": "human", "scale": args.scale, "reads": rs.n_reads, "genome_bp": rs.meta["genome"],
           "kmers": n_kmers, "refine": refine, "fine_partitions": b.np, "fine_p": fine_p,
           "ranges": len(res.ranges), "batches": res.batches, "resident": args.resident,
           "h2d_gb": res.h2d_bytes / 1e9, "stream_wall_s": wall_s, "stream_device_ms": dev_ms,
           "kmers_per_s_wall": n_kmers / wall_s, "stats": st, "gen_s": gen_s, "encode_s": enc_s,
           "I1": st["sum_count"] == n_kmers, "I2": st["sum_edges"] == 2 * int(np.maximum(L - k, 0).sum())}
    g = np.concatenate(kept) if kept else np.zeros(0, dtype=VERTEX_DTYPE)
    g = g[np.lexsort((g["kmer_lo"], g["kmer_hi"]))]
    out["sampled_pids"] = pids.tolist()
    out["sampled_vertices"] = int(len(g))
    if not args.no_oracle:
        t3 = time.time()
        orc = oracle.graph(rs.seq, rs.offsets, k, p, np_, n_threads=os.cpu_count() or 1, pids=pids.tolist())
        out["oracle_s"] = time.time() - t3
        ok = len(g) == len(orc) and np.array_equal(g["kmer_hi"], orc["key_hi"]) and \
            np.array_equal(g["kmer_lo"], orc["key_lo"]) and \
            all(np.array_equal(g[f], orc[f]) for f in ("count", "out", "in", "pid"))
        out["sampled_parity"] = bool(ok)
        out["oracle_vertices"] = int(len(orc))
    print(json.dumps(out), flush=True)
    return 0 if out["I1"] and out["I2"] and out.get("sampled_parity", True) else 1


if __name__ == "__main__":
    sys.exit(main())

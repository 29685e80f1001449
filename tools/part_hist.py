"""Partition-size distribution of a config after MSP (fraction of K-mers in partitions above a size)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from synth import make_config
from paper_conf_icdcs_qiul17_b200 import DbgBuilder, encode_reads

name = sys.argv[1] if len(sys.argv) > 1 else "ecoli"
rs = make_config(name)
for refine in (1, 32, 256, 1024):
    b = DbgBuilder(rs.k, rs.p, rs.num_partitions, refine=refine)
    d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
    b.msp(d_bases, d_off)
    pk = b.part_kmers
    tot = pk.sum()
    s = np.sort(pk)[::-1]
    line = f"refine {refine:5d} NPF {b.np:8d} mean {pk.mean():9.1f} max {s[0]:9d} p99 {np.percentile(pk, 99):9.1f}"
    for thr in (960, 1600, 3300, 6592, 20000):
        line += f" | >{thr}: {pk[pk > thr].sum() / tot * 100:5.1f}%"
    print(line, flush=True)

import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle
from synth import genome, make_reads, ReadSet
from paper_conf_icdcs_qiul17_b200 import build_graph, DbgBuilder, encode_reads, _lib

k, p, np_, refine = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
g = genome(60_000, seed=k + np_)
seq, offs = make_reads(g, 4000, 100, 0.01, seed=refine + 3)
rs = ReadSet(seq, offs)
orc = oracle.graph(rs.seq, rs.offsets, k, p, np_, n_threads=os.cpu_count())
for mode in ("smem", "resident"):
    res = build_graph(rs.seq, rs.offsets, k, p, np_, refine=refine, mode=mode)
    v = res.vertices
    bad = np.nonzero((v["count"] != orc["count"]))[0]
    print(mode, "n", len(v), len(orc), "bad", len(bad), "batches", res.batches)
    for i in bad[:4]:
        print("  gpu", v[i], "\n  orc", orc[i])
b = DbgBuilder(k, p, np_, refine=refine)
d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
b.msp(d_bases, d_off)
slots = _lib.dbg_smem_table_slots(b.prm)
caps = np.array([_lib.dbg_table_capacity(b.prm, int(n)) for n in b.part_kmers])
print("slots", slots, "caps", sorted(caps)[-5:], "n off-chip", int((caps > slots).sum()))

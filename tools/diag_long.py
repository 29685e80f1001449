import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch
import oracle
from synth import random_reads, ReadSet
from paper_conf_icdcs_qiul17_b200 import DbgBuilder, encode_reads, build_graph, _lib
from gpu_helpers import decode_records, occurrences_from_records, occurrences_from_oracle_msp

def readset(reads):
    b = "".join(reads).encode()
    offs = np.zeros(len(reads) + 1, dtype=np.uint64)
    offs[1:] = np.cumsum([len(r) for r in reads])
    return ReadSet(np.frombuffer(b, dtype=np.uint8).copy(), offs)

k, p, np_ = 9, 3, 13
rs = random_reads(20, 300, 3000, seed=7 + k)
reads = rs.reads() + ["A" * 700, "AC" * 400, "ACGTTGCA" * 90, "T" * (k + 1), "G" * k, "ACG"]
rs = readset(reads)
b = DbgBuilder(k, p, np_)
d_bases, d_off = b.upload(encode_reads(rs.seq), rs.offsets)
b.msp(d_bases, d_off)
torch.cuda.synchronize()
sk = oracle.msp(rs.seq, rs.offsets, k, p, np_)
want_k = np.bincount(sk["pid"], weights=sk["n_kmers"], minlength=np_).astype(np.int64)
print("part_kmers", b.part_kmers.tolist())
print("want_k    ", want_k.tolist())
nrec = int(b.part_records.sum())
words = b.records[: nrec * b.rec_words].cpu().numpy().view(np.uint32)
recs = decode_records(words, b.rec_words, k)
a1 = occurrences_from_records(recs, k); a2 = occurrences_from_oracle_msp(sk, rs.reads(), k)
print("msp occurrences equal:", a1 == a2)
orc = oracle.graph(rs.seq, rs.offsets, k, p, np_)
print("distinct per pid", np.bincount(orc["pid"], minlength=np_).tolist())
for mode in ("resident", "fused"):
    try:
        r = build_graph(rs.seq, rs.offsets, k, p, np_, mode=mode)
        print(mode, "ok", r.n_vertices, len(orc))
    except Exception as e:
        print(mode, "FAIL", e)

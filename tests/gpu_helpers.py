"""Test-side helpers for GPU parity (decoding records, comparing with the oracle)."""
from collections import Counter

import numpy as np

FIELDS = ("count", "out", "in", "pid")


def compare_vertices(gpu, orc):
    """Bit-exact comparison of sorted GPU dbg_vertex records with oracle records."""
    assert len(gpu) == len(orc), (len(gpu), len(orc))
    assert np.array_equal(gpu["kmer_hi"], orc["key_hi"])
    assert np.array_equal(gpu["kmer_lo"], orc["key_lo"])
    for f in FIELDS:
        if not np.array_equal(gpu[f], orc[f]):
            bad = np.nonzero((gpu[f] != orc[f]).reshape(len(gpu), -1).any(axis=1))[0][:5]
            raise AssertionError(f"field {f} differs at {bad}: gpu={gpu[bad]} oracle={orc[bad]}")


def decode_records(words: np.ndarray, rec_words: int, k: int):
    """Records (dbg.h layout) -> list of (pid, bases string, n_kmers, has_left, has_right)."""
    w = words.reshape(-1, rec_words).astype(np.uint64)
    out = []
    for row in w:
        hdr = int(row[0])
        n, hl, hr, pid = hdr & 63, (hdr >> 6) & 1, (hdr >> 7) & 1, hdr >> 8
        nb = hl + n + k - 1 + hr
        bases = []
        for i in range(nb):
            word = int(row[1 + i // 16])
            bases.append("ACGT"[(word >> (30 - 2 * (i % 16))) & 3])
        out.append((pid, "".join(bases), n, hl, hr))
    return out


def occurrences_from_records(recs, k):
    """Per-pid Counter of (kmer, pred, succ) occurrences from decoded records."""
    per = {}
    for pid, s, n, hl, hr in recs:
        c = per.setdefault(pid, Counter())
        for t in range(n):
            i = hl + t
            pred = s[i - 1] if i > 0 else None
            succ = s[i + k] if i + k < len(s) else None
            c[(s[i:i + k], pred, succ)] += 1
    return per


def occurrences_from_oracle_msp(sk, reads, k):
    norm = str.maketrans("acgtn", "ACGTA")
    per = {}
    for row in sk:
        r = "".join(ch if ch in "ACGT" else "A" for ch in reads[int(row["read"])].translate(norm))
        c = per.setdefault(int(row["pid"]), Counter())
        for t in range(int(row["n_kmers"])):
            i = int(row["start"]) + t
            pred = r[i - 1] if i > 0 else None
            succ = r[i + k] if i + k < len(r) else None
            c[(r[i:i + k], pred, succ)] += 1
    return per

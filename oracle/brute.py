"""Pure-Python string brute force -- TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Used to pin the C++ oracle on tiny inputs.  Everything is done on Python
strings: canonical = lexicographically smaller string of (x, rc(x)) (PAPER.md
L197-201), minimizer = min() over the window's canonical P-mer strings
(Definition 1), partition = fmix64(code) mod NP (Sec. III-B
L455-459, reading I), and the bi-directed edge rule of SURVEY.md 8(c) steps 6-7.
It shares no code with dbg_oracle.cpp (different language, string compare
instead of integer codes).
"""
from __future__ import annotations

from collections import defaultdict

_COMP = str.maketrans("ACGT", "TGCA")
_ORDER = "ACGT"
M64 = (1 << 64) - 1


def normalise(read: str) -> str:
    """Sec. II-A: unknown characters become 'A' (lower case -> upper, reading B)."""
    return "".join(c if c in "ACGT" else "A" for c in read.upper())


def rc(s: str) -> str:
    return s.translate(_COMP)[::-1]


def code(s: str) -> int:
    """Integer value with the first base most significant, A=0 C=1 G=2 T=3 (reading A)."""
    v = 0
    for c in s:
        v = v * 4 + _ORDER.index(c)
    return v


def fmix64(k: int) -> int:
    k &= M64
    k ^= k >> 33
    k = (k * 0xFF51AFD7ED558CCD) & M64
    k ^= k >> 33
    k = (k * 0xC4CEB9FE1A85EC53) & M64
    k ^= k >> 33
    return k


def canonical_string(x: str) -> str:
    y = rc(x)
    return x if x <= y else y


def minimizer_string(kmer: str, p: int) -> str:
    """Definition 1 with readings D/E: smallest canonical P-substring of the K-mer."""
    return min(canonical_string(kmer[j:j + p]) for j in range(len(kmer) - p + 1))


def partition(kmer: str, p: int, num_partitions: int) -> int:
    return fmix64(code(minimizer_string(kmer, p))) % num_partitions


def graph(reads, k: int, p: int, num_partitions: int):
    """dict canonical-string -> [count, out[4], in[4], pid]."""
    g = {}
    for raw in reads:
        s = normalise(raw)
        for i in range(len(s) - k + 1):
            x = s[i:i + k]
            v = canonical_string(x)
            fwd = x <= rc(x)
            pid = partition(x, p, num_partitions)
            e = g.setdefault(v, [0, [0, 0, 0, 0], [0, 0, 0, 0], pid])
            if e[3] != pid:
                raise AssertionError("vertex in two partitions")
            e[0] += 1
            pred = s[i - 1] if i > 0 else None
            succ = s[i + k] if i + k < len(s) else None
            if fwd:
                if succ:
                    e[1][_ORDER.index(succ)] += 1
                if pred:
                    e[2][_ORDER.index(pred)] += 1
            else:
                # the vertex is rc(x): x's successor c precedes rc(x) as comp(c), and
                # x's predecessor c follows rc(x) as comp(c)
                if succ:
                    e[2][_ORDER.index(rc(succ))] += 1
                if pred:
                    e[1][_ORDER.index(rc(pred))] += 1
    return g


def superkmers(reads, k: int, p: int, num_partitions: int):
    """List of (read, start, n_kmers, pid, has_left, has_right, minimizer-string)."""
    out = []
    for r, raw in enumerate(reads):
        s = normalise(raw)
        nk = len(s) - k + 1
        if nk <= 0:
            continue
        m = [minimizer_string(s[i:i + k], p) for i in range(nk)]
        start = 0
        for i in range(1, nk + 1):
            if i == nk or m[i] != m[start]:
                pid = fmix64(code(m[start])) % num_partitions
                out.append((r, start, i - start, pid, int(start > 0), int(i - 1 + k < len(s)), m[start]))
                start = i
    return out


def kplus1_closed_form(reads, k: int):
    """Independent closed form over (K+1)-mer / K-mer occurrence counts (odd K only).

    count_v = occ(v) + occ(rc v); out_v[c] = occ(v.c) + occ(rc(v.c));
    in_v[c] = occ(c.v) + occ(rc(c.v)), with occ counted on the reads as given.
    Returns dict canonical-string -> [count, out[4], in[4]] (no pid).
    """
    occ_k = defaultdict(int)
    occ_k1 = defaultdict(int)
    for raw in reads:
        s = normalise(raw)
        for i in range(len(s) - k + 1):
            occ_k[s[i:i + k]] += 1
        for i in range(len(s) - k):
            occ_k1[s[i:i + k + 1]] += 1
    verts = {canonical_string(x) for x in occ_k}
    g = {}
    for v in verts:
        cnt = occ_k[v] + (occ_k[rc(v)] if rc(v) != v else 0)
        out = []
        inn = []
        for c in _ORDER:
            a = v + c
            b = c + v
            out.append(occ_k1[a] + occ_k1[rc(a)])
            inn.append(occ_k1[b] + occ_k1[rc(b)])
        g[v] = [cnt, out, inn]
    return g
